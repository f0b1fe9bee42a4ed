"""Seeded synthetic input generators shared by the tests, the oracle side and bench.py.

Holds NO arithmetic of the method (no field, curve or MSM code): it only draws
random numbers.  Curve-dependent bounds (r, λ) are passed in by the caller.

Input recipe:
  * scalars k_i uniform on [0, r): S = ceil(λ/32) little-endian u32 words each, the top
    word masked to λ bits, values >= r redrawn (numpy PCG64, fixed seed);
  * point seeds (e0, delta) uniform on [1, r): the points are P_i = (e0 + i*delta) G,
    computed by whoever needs them (the oracle for small n; the library's generator
    kernel for bench sizes) — random (e0, delta) make accidental exceptional cases
    (P == ±acc inside a bucket) need linear relations with coefficients ~ r;
  * adversarial scalar patterns for edge-case tests.
"""
import numpy as np


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def words_ge(x: np.ndarray, bound_words: np.ndarray) -> np.ndarray:
    """Row-wise x >= bound for little-endian u32 word rows (vectorised compare)."""
    n, S = x.shape
    ge = np.ones(n, dtype=bool)      # equal so far => >=
    decided = np.zeros(n, dtype=bool)
    for w in range(S - 1, -1, -1):
        gt = (x[:, w] > bound_words[w]) & ~decided
        lt = (x[:, w] < bound_words[w]) & ~decided
        ge[gt] = True
        ge[lt] = False
        decided |= gt | lt
    return ge


def int_to_words(v: int, S: int) -> np.ndarray:
    return np.array([(v >> (32 * i)) & 0xFFFFFFFF for i in range(S)], dtype=np.uint32)


def scalars(r: int, n: int, seed: int) -> np.ndarray:
    """n scalars uniform on [0, r) as an [n, S] uint32 array (little-endian words)."""
    lam = r.bit_length()
    S = (lam + 31) // 32
    top_bits = lam - 32 * (S - 1)
    top_mask = np.uint32((1 << top_bits) - 1)
    rw = int_to_words(r, S)
    g = _rng(seed)
    out = np.empty((n, S), dtype=np.uint32)
    todo = np.arange(n)
    while todo.size:
        x = g.integers(0, 1 << 32, size=(todo.size, S), dtype=np.uint64).astype(np.uint32)
        x[:, S - 1] &= top_mask
        ok = ~words_ge(x, rw)
        out[todo[ok]] = x[ok]
        todo = todo[~ok]
    return out


def point_seeds(r: int, seed: int) -> tuple[int, int]:
    """(e0, delta) uniform on [1, r)."""
    g = _rng(seed ^ 0x5EED5EED)
    lam = r.bit_length()

    def draw():
        while True:
            v = 0
            for _ in range((lam + 31) // 32):
                v = (v << 32) | int(g.integers(0, 1 << 32, dtype=np.uint64))
            v &= (1 << lam) - 1
            if 1 <= v < r:
                return v
    return draw(), draw()


def words_to_ints(a: np.ndarray) -> list[int]:
    """[n, S] little-endian u32 rows -> Python ints (test/oracle convenience)."""
    a = np.ascontiguousarray(a, dtype=np.uint32)
    S = a.shape[1]
    b = a.view(np.uint8).reshape(a.shape[0], 4 * S)
    return [int.from_bytes(row.tobytes(), "little") for row in b]


def ints_to_words(vals, S: int) -> np.ndarray:
    out = np.zeros((len(vals), S), dtype=np.uint32)
    for i, v in enumerate(vals):
        out[i] = int_to_words(v, S)
    return out


def pattern_scalars(r: int, n: int, seed: int, kind: str) -> np.ndarray:
    """Adversarial scalar patterns (edge cases, R19)."""
    lam = r.bit_length()
    S = (lam + 31) // 32
    g = _rng(seed)
    if kind == "zeros":
        vals = [0] * n
    elif kind == "ones":
        vals = [1] * n
    elif kind == "max":
        vals = [r - 1] * n
    elif kind == "equal":
        v = int(g.integers(1, 1 << 62))
        vals = [v] * n
    elif kind == "skewed":      # 90 % of scalars in {0, 1, 2}, rest uniform
        u = scalars(r, n, seed)
        small = g.random(n) < 0.9
        sv = g.integers(0, 3, size=n)
        vals = [int(sv[i]) if small[i] else None for i in range(n)]
        uu = words_to_ints(u)
        vals = [uu[i] if v is None else v for i, v in enumerate(vals)]
    elif kind == "extremes":    # 0, 1, r-1, 2^(λ-1), 2^(λ-1)-1, r-2, ... cycled
        ex = [0, 1, r - 1, 1 << (lam - 1), (1 << (lam - 1)) - 1, r - 2, 2, (1 << (lam - 2))]
        vals = [ex[i % len(ex)] for i in range(n)]
    else:
        raise ValueError(kind)
    return ints_to_words(vals, S)


SCALAR_CHUNK = 1 << 20


def scalars_range(r: int, start: int, count: int, seed: int) -> np.ndarray:
    """Rows [start, start+count) of an arbitrarily long uniform scalar vector: chunk t of
    SCALAR_CHUNK rows is drawn from seed (seed, t), so any slice (a rank's shard) is
    generated independently and identically for every world size."""
    lam = r.bit_length()
    S = (lam + 31) // 32
    out = np.empty((count, S), dtype=np.uint32)
    t0 = start // SCALAR_CHUNK
    t1 = (start + count + SCALAR_CHUNK - 1) // SCALAR_CHUNK
    for t in range(t0, t1):
        lo = max(start, t * SCALAR_CHUNK)
        hi = min(start + count, (t + 1) * SCALAR_CHUNK)
        if hi <= lo:
            continue
        chunk = scalars(r, SCALAR_CHUNK, (seed * 1000003 + t) & 0x7FFFFFFFFFFFFFFF)
        out[lo - start:hi - start] = chunk[lo - t * SCALAR_CHUNK:hi - t * SCALAR_CHUNK]
    return out


def progression_offset(r: int, e0: int, delta: int, off: int) -> int:
    """e_off = e0 + off*delta mod r: the first point scalar of a shard starting at `off`
    (input bookkeeping for the generator, not curve arithmetic)."""
    return (e0 + off * delta) % r


# Scalar-field orders r (bit length = λ, Table 1): the range of the uniform scalar
# draw.  Constants of the input recipe, not arithmetic; the oracle keeps its own copy in
# oracle/curves.py and the library its own in csrc/params.h.
CURVE_ORDERS = {
    "bn254": 0x30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001,
    "bls12_377": 0x12ab655e9a2ca55660b44d1e5c37b00159aa76fed00000010a11800000000001,
    "bls12_381": 0x73eda753299d7d483339d80809a1d80553bda402fffe5bfeffffffff00000001,
    "mnt4_753": 0x01c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db26c5c28c859a99b3eebca9429212636b9dff97634993aa4d6c381bc3f0057974ea099170fa13a4fd90776e240000001,
}
