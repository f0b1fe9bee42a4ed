"""Test helpers: limb packing and cached oracle-generated inputs (test side only)."""
import functools

import numpy as np

import synth
from oracle import points as opoints
from oracle.curves import CURVES

L32 = {"bn254": 8, "bls12_377": 12, "bls12_381": 12, "mnt4_753": 24}
S_W = {"bn254": 8, "bls12_377": 8, "bls12_381": 8, "mnt4_753": 24}


def to_words(v: int, nw: int) -> np.ndarray:
    return np.array([(v >> (32 * i)) & 0xFFFFFFFF for i in range(nw)], dtype=np.uint32)


def from_words(ws) -> int:
    return int.from_bytes(np.asarray(ws, dtype=np.uint32).tobytes(), "little")


def points_to_words(Ps, name) -> np.ndarray:
    w = L32[name]
    out = np.zeros((len(Ps), 2 * w), dtype=np.uint32)
    for i, P in enumerate(Ps):
        if P is not None:
            out[i, :w] = to_words(P[0], w)
            out[i, w:] = to_words(P[1], w)
    return out


def words_to_point(ws, name):
    w = L32[name]
    x, y = from_words(ws[:w]), from_words(ws[w:2 * w])
    return None if (x, y) == (0, 0) else (x, y)


@functools.lru_cache(maxsize=64)
def progression(name: str, n: int, seed: int):
    """(points, e_i) for P_i = (e0 + i*delta) G, from the oracle (cached per process)."""
    c = CURVES[name]
    e0, d = synth.point_seeds(c.r, seed)
    Ps = opoints.progression_points(e0, d, n, c)
    es = opoints.progression_scalars(e0, d, n, c)
    return tuple(Ps), tuple(es), e0, d
