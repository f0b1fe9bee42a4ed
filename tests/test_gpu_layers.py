"""GPU parity of the field and EC layers and of the digit decomposition, through the
C-ABI debug entry points, against the oracle / plain definitions."""
import random

import numpy as np
import pytest

import synth
from oracle import ec, stages
from oracle.curves import CURVES
from tests.helpers import L32, S_W, points_to_words, progression, to_words, words_to_point, from_words

pytestmark = pytest.mark.gpu
NAMES = ["bn254", "bls12_377", "bls12_381", "mnt4_753"]


@pytest.fixture(scope="module")
def msm():
    from paper_conf_asplos_ji0x024_b200 import msm as m
    assert m.device_count() >= 1, "no CUDA device"
    return m


def field_vals(c, n, seed):
    rng = random.Random(seed)
    W = {"bn254": 30, "bls12_377": 30, "bls12_381": 30, "mnt4_753": 29}
    edge = [0, 1, 2, c.p - 1, c.p - 2, (c.p - 1) // 2, (1 << (c.pbits - 1)), (1 << 32) - 1, (1 << 30) - 1,
            (1 << 30), c.p - (1 << 30)]
    return edge + [rng.randrange(c.p) for _ in range(n - len(edge))]


@pytest.mark.parametrize("name", NAMES)
def test_field_ops(msm, name):
    c = CURVES[name]
    w = L32[name]
    n = 2048 if name != "mnt4_753" else 512
    A = field_vals(c, n, 1)
    B = list(reversed(field_vals(c, n, 2)))
    a = np.stack([to_words(v, w) for v in A])
    b = np.stack([to_words(v, w) for v in B])
    p = c.p
    exp = {
        0: [x * y % p for x, y in zip(A, B)],
        1: [x * x % p for x in A],
        2: [(x + y) % p for x, y in zip(A, B)],
        3: [(x - y) % p for x, y in zip(A, B)],
        5: [(-x) % p for x in A],
        7: [2 * x * y % p for x, y in zip(A, B)],      # fmul_sum(a, b, b, a)
        8: [x * (y + x) % p for x, y in zip(A, B)],    # fmul_sum(a, b, a, a)
    }
    for op, want in exp.items():
        got = msm.debug_field(name, op, a, b)
        bad = [i for i in range(n) if from_words(got[i]) != want[i]]
        assert not bad, (op, bad[:5])
    # inversion (non-zero inputs)
    nz = [v if v else 1 for v in A[:256]]
    a2 = np.stack([to_words(v, w) for v in nz])
    got = msm.debug_field(name, 4, a2, a2)
    assert all(from_words(got[i]) == pow(nz[i], -1, p) for i in range(len(nz)))
    # binary-GCD inversion (the final normalisation's): every non-zero edge value and
    # random values; 0 maps to 0 (no inverse) instead of looping
    got = msm.debug_field(name, 6, a2, a2)
    assert all(from_words(got[i]) == pow(nz[i], -1, p) for i in range(len(nz)))
    z = np.zeros((4, w), dtype=np.uint32)
    assert not msm.debug_field(name, 6, z, z).any()


def _z_words(c, n, seed):
    rng = random.Random(seed)
    w = L32[c.name]
    z = np.zeros((n, 2 * w), dtype=np.uint32)
    for i in range(n):
        z[i, :w] = to_words(rng.randrange(1, c.p), w)
        z[i, w:] = to_words(rng.randrange(1, c.p), w)
    return z


@pytest.mark.parametrize("name", NAMES)
def test_ec_ops_and_exceptional_cases(msm, name):
    c = CURVES[name]
    Ps, _, _, _ = progression(name, 24, 11)
    Ps = list(Ps)
    P = Ps[:12]
    Q = Ps[12:24]
    # exceptional pairs appended: equal, opposite, O operands
    P += [Ps[0], Ps[1], None, Ps[2], None]
    Q += [Ps[0], ec.neg(Ps[1], c), Ps[3], None, None]
    n = len(P)
    Pw, Qw = points_to_words(P, name), points_to_words(Q, name)
    z = _z_words(c, n, 5)
    got_acc = msm.debug_ec(name, 0, Pw, Qw, z)
    got_add = msm.debug_ec(name, 1, Pw, Qw, z)
    got_dbl = msm.debug_ec(name, 2, Pw, Qw, z)
    for i in range(n):
        want = ec.add(P[i], Q[i], c)
        assert words_to_point(got_acc[i], name) == want, ("acc", i)
        assert words_to_point(got_add[i], name) == want, ("add", i)
        assert words_to_point(got_dbl[i], name) == ec.double(P[i], c), ("dbl", i)


@pytest.mark.parametrize("name", NAMES)
def test_signed_digits(msm, name):
    c = CURVES[name]
    ks = synth.words_to_ints(synth.scalars(c.r, 200, 3)) + \
        synth.words_to_ints(synth.pattern_scalars(c.r, 16, 4, "extremes"))
    sw = synth.ints_to_words(ks, S_W[name])
    for cc in (2, 3, 5, 8, 13, 16, 21, 24):
        got = msm.debug_digits(name, cc, sw)
        for i, k in enumerate(ks):
            assert list(got[i]) == stages.signed_digits(k, c.lam, cc), (cc, i)
