"""Pins for oracle/ec.py and oracle/xyzz.py: group laws (closed under the curve,
identity, inverse, associativity, commutativity), scalar-multiplication linearity,
and the XYZZ formulas of Alg. 1 / Alg. 4 / PDBL against affine Formula (1),
including the exceptional cases."""
import random

import pytest

from oracle import ec, xyzz
from oracle.curves import CURVES

ALL = list(CURVES.values())


def rand_points(c, k, seed):
    rng = random.Random(seed)
    return [ec.mul(rng.randrange(1, c.r), c.G, c) for _ in range(k)]


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_group_laws(c):
    P, Q, S = rand_points(c, 3, 1)
    for X in (P, Q, S):
        assert ec.on_curve(X, c)
    assert ec.add(P, None, c) == P and ec.add(None, P, c) == P
    assert ec.add(P, ec.neg(P, c), c) is None
    assert ec.add(P, Q, c) == ec.add(Q, P, c)
    assert ec.add(ec.add(P, Q, c), S, c) == ec.add(P, ec.add(Q, S, c), c)
    assert ec.add(P, P, c) == ec.double(P, c)
    assert ec.on_curve(ec.add(P, Q, c), c) and ec.on_curve(ec.double(P, c), c)


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_scalar_mul_linearity(c):
    rng = random.Random(2)
    P = rand_points(c, 1, 5)[0]
    a, b = rng.randrange(c.r), rng.randrange(c.r)
    assert ec.mul(a + b, P, c) == ec.add(ec.mul(a, P, c), ec.mul(b, P, c), c)
    assert ec.mul(a * b % c.r, P, c) == ec.mul(a, ec.mul(b, P, c), c)
    # small k by repeated addition (brute force)
    R = None
    for k in range(0, 9):
        assert ec.mul(k, P, c) == R
        R = ec.add(R, P, c)


def _xyzz_scale(A, z, c):
    """Same point, different representative: (X z^2, Y z^3, ZZ z^2, ZZZ z^3)."""
    X, Y, ZZ, ZZZ = A
    p = c.p
    return (X * z * z % p, Y * z**3 % p, ZZ * z * z % p, ZZZ * z**3 % p)


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_xyzz_formulas_match_affine(c):
    rng = random.Random(11)
    P, Q = rand_points(c, 2, 9)
    A = _xyzz_scale(xyzz.from_affine(P), rng.randrange(2, c.p), c)
    B = _xyzz_scale(xyzz.from_affine(Q), rng.randrange(2, c.p), c)
    assert xyzz.to_affine(xyzz.padd(A, B, c), c) == ec.add(P, Q, c)
    assert xyzz.to_affine(xyzz.pacc(A, Q, c), c) == ec.add(P, Q, c)
    assert xyzz.to_affine(xyzz.pdbl(A, c), c) == ec.double(P, c)
    # exceptional cases (R7)
    assert xyzz.to_affine(xyzz.pacc(A, P, c), c) == ec.double(P, c)             # P == acc
    assert xyzz.to_affine(xyzz.pacc(A, ec.neg(P, c), c), c) is None            # P == -acc
    assert xyzz.pacc(xyzz.O, Q, c) == (Q[0], Q[1], 1, 1)                         # acc == O
    assert xyzz.pacc(A, None, c) == A
    assert xyzz.to_affine(xyzz.padd(A, _xyzz_scale(A, 5, c), c), c) == ec.double(P, c)
    assert xyzz.to_affine(xyzz.padd(A, xyzz.from_affine(ec.neg(P, c)), c), c) is None
    assert xyzz.padd(xyzz.O, B, c) == B and xyzz.padd(A, xyzz.O, c) == A
    assert xyzz.pdbl(xyzz.O, c) == xyzz.O


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_xyzz_invariant(c):
    """ZZ^3 == ZZZ^2 is preserved by every formula."""
    P, Q = rand_points(c, 2, 21)
    A = xyzz.from_affine(P)
    for _ in range(3):
        A = xyzz.pacc(A, Q, c)
        A = xyzz.padd(A, A if False else xyzz.pdbl(A, c), c)
        X, Y, ZZ, ZZZ = A
        assert pow(ZZ, 3, c.p) == pow(ZZZ, 2, c.p)
