"""Pins for oracle/field.py: Alg. 2 (SOS) against the closed form A*B*R^-1 mod n."""
import random

import pytest

from oracle.curves import CURVES
from oracle.field import from_words, inv, mont_mul_sos, n0_prime, to_words

ALL = list(CURVES.values())


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_n0_prime(c):
    assert (c.p * n0_prime(c.p)) % (1 << 32) == (1 << 32) - 1


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_sos_matches_definition(c):
    rng = random.Random(7)
    N = c.L
    R = 1 << (32 * N)
    Rinv = inv(R, c.p)
    edge = [0, 1, 2, c.p - 1, c.p - 2, R % c.p, (R - 1) % c.p, (1 << (c.pbits - 1))]
    vals = edge + [rng.randrange(c.p) for _ in range(40)]
    for a in vals:
        b = rng.choice(vals)
        assert mont_mul_sos(a, b, c.p, N) == a * b * Rinv % c.p


def test_sos_round_trip_montgomery_form():
    c = CURVES["bls12_381"]
    R = 1 << (32 * c.L)
    rng = random.Random(3)
    for _ in range(20):
        a, b = rng.randrange(c.p), rng.randrange(c.p)
        am, bm = a * R % c.p, b * R % c.p
        prod_m = mont_mul_sos(am, bm, c.p, c.L)
        assert mont_mul_sos(prod_m, 1, c.p, c.L) == a * b % c.p


def test_words_roundtrip():
    x = (1 << 381) - 12345
    assert from_words(to_words(x, 12)) == x
