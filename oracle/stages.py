"""The staged decomposition the GPU path uses, written plainly (test infrastructure only).

This is the oracle for stage-level parity: every intermediate here is a unique
group element (or integer) once the window size c and the digit rule are fixed,
so the GPU's bucket sums and window sums can be compared one by one.

Signed-digit rule (PAPER.md:428 adopts signed digits without stating a rule;
DESIGN.md reading R6):
    nwin = floor(λ / c) + 1
    chunk_j = bits [j c, j c + c) of k;  d_j = chunk_j + carry_j
    for j < nwin-1: if d_j > 2^(c-1): d_j -= 2^c, carry_{j+1} = 1 else carry_{j+1} = 0
    the top digit is never negated.
    => k = sum_j d_j 2^(j c), d_j in (-2^(c-1), 2^(c-1)] (top digit in [0, 2^(c-1)]).
Bucket of a digit: |d_j| in [0, 2^(c-1)] (0 = no bucket), sign = d_j < 0 (the point
is negated, y -> p - y).

B_{j,b} = sum_{i : |d_ij| = b} sgn(d_ij) P_i                 (bucket-sum)
W_j     = sum_{b=1}^{2^(c-1)} b * B_{j,b}                     (bucket-reduce, PAPER.md:143, 161;
                                                             "2^i B_i" read as b*B_b, R12)
Q       = sum_j 2^(j c) W_j  by Horner                        (window-reduce)

With precomputation ("For a given point P_i, values such as 2^s P_i,
2^{2s} P_i, and so on, are precomputed. As a result, in window j, the point P_i is
replaced with 2^{js} P_i"; "bucket-reduce and window-reduce are commutative
with precomputation") all windows share ONE bucket set:
T_{j,i}  = 2^(j c) P_i                                        (table row j: c doublings of row j-1)
B^pre_b  = sum_{(i,j) : |d_ij| = b} sgn(d_ij) T_{j,i}
Q        = sum_{b=1}^{2^(c-1)} b * B^pre_b                    (one bucket-reduce, no window-reduce)
"""
from . import ec


def num_windows(lam: int, c: int) -> int:
    return lam // c + 1


def signed_digits(k: int, lam: int, c: int) -> list[int]:
    assert 0 <= k < (1 << lam)
    nwin = num_windows(lam, c)
    half = 1 << (c - 1)
    mask = (1 << c) - 1
    out = []
    carry = 0
    for j in range(nwin):
        d = ((k >> (j * c)) & mask) + carry
        if j < nwin - 1 and d > half:
            d -= 1 << c
            carry = 1
        else:
            carry = 0
        out.append(d)
    return out


def bucket_sums(ks, Ps, c, curve):
    """Returns B[j][b] (affine, None = O) for b in 0..2^(c-1) (B[j][0] unused = None)."""
    nwin = num_windows(curve.lam, c)
    nb = (1 << (c - 1)) + 1
    B = [[None] * nb for _ in range(nwin)]
    for k, P in zip(ks, Ps):
        ds = signed_digits(k, curve.lam, c)
        for j, d in enumerate(ds):
            if d == 0:
                continue
            Q = P if d > 0 else ec.neg(P, curve)
            B[j][abs(d)] = ec.add(B[j][abs(d)], Q, curve)
    return B


def window_sums(B, curve):
    """W_j = sum_b b * B_{j,b}, by the descending running sum."""
    W = []
    for Bj in B:
        running = None
        Wj = None
        for b in range(len(Bj) - 1, 0, -1):
            running = ec.add(running, Bj[b], curve)
            Wj = ec.add(Wj, running, curve)
        W.append(Wj)
    return W


def window_combine(W, c, curve):
    """Q = sum_j 2^(j c) W_j by Horner: c PDBL per window step."""
    Q = None
    for j in range(len(W) - 1, -1, -1):
        for _ in range(c):
            Q = ec.double(Q, curve)
        Q = ec.add(Q, W[j], curve)
    return Q


def msm_staged(ks, Ps, c, curve):
    return window_combine(window_sums(bucket_sums(ks, Ps, c, curve), curve), c, curve)


def precomputed_table(Ps, c, curve):
    """T[j][i] = 2^(j c) P_i for j < nwin, each row c doublings of the previous one."""
    nwin = num_windows(curve.lam, c)
    T = [list(Ps)]
    for _ in range(1, nwin):
        row = []
        for P in T[-1]:
            for _ in range(c):
                P = ec.double(P, curve)
            row.append(P)
        T.append(row)
    return T


def bucket_sums_precomputed(ks, Ps, c, curve):
    """B^pre[b] (affine, None = O), b in 0..2^(c-1): one shared bucket set over all windows."""
    T = precomputed_table(Ps, c, curve)
    nb = (1 << (c - 1)) + 1
    B = [None] * nb
    for i, k in enumerate(ks):
        for j, d in enumerate(signed_digits(k, curve.lam, c)):
            if d == 0:
                continue
            Q = T[j][i] if d > 0 else ec.neg(T[j][i], curve)
            B[abs(d)] = ec.add(B[abs(d)], Q, curve)
    return B


def msm_precomputed(ks, Ps, c, curve):
    """Q = sum_b b * B^pre_b (a single bucket-reduce)."""
    return window_sums([bucket_sums_precomputed(ks, Ps, c, curve)], curve)[0]


def bucket_split_partial(ks, Ps, c, curve, G, g, pre=False):
    """Part g of G of the bucket split (§3.2.2: DistMSM "splits the buckets
    into GPUs-per-window parts"; each GPU reduces only its buckets and the CPU adds the
    N_gpu results).  Part g owns the buckets b = |d| with b mod G = g
    (reading R18: interleaved, so the top window's small digits spread over all
    parts).  Written from the definitions, not the running sum:
        without the table:  sum_j 2^(j c) * sum_{b mod G = g} b * B_{j,b}
        with it (pre):      sum_{b mod G = g} b * B^pre_b
    The G parts sum to Q."""
    if pre:
        B = bucket_sums_precomputed(ks, Ps, c, curve)
        Q = None
        for b in range(1, len(B)):
            if b % G == g:
                Q = ec.add(Q, ec.mul(b, B[b], curve), curve)
        return Q
    Bw = bucket_sums(ks, Ps, c, curve)
    Q = None
    for j, Bj in enumerate(Bw):
        Wj = None
        for b in range(1, len(Bj)):
            if b % G == g:
                Wj = ec.add(Wj, ec.mul(b, Bj[b], curve), curve)
        Q = ec.add(Q, ec.mul(1 << (j * c), Wj, curve), curve)
    return Q
