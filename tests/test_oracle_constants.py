"""Pins for oracle/curves.py: the constants are checked against what the
mathematics fixes, not against another copy of themselves."""
import json
import os

import pytest
import sympy

from oracle import ec
from oracle.curves import CURVES

GOLD = os.path.join(os.path.dirname(__file__), "golden")
ALL = list(CURVES.values())


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_primes(c):
    assert sympy.isprime(c.p)
    assert sympy.isprime(c.r)


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_table1_bit_widths(c):
    t = json.load(open(os.path.join(GOLD, "table1_bits.json")))
    assert c.lam == t["k_bits"][c.name]
    assert c.pbits == t["P_bits"][c.name]


def test_family_closed_forms():
    bn = CURVES["bn254"]
    u = bn.u
    assert bn.p == 36 * u**4 + 36 * u**3 + 24 * u**2 + 6 * u + 1
    assert bn.r == 36 * u**4 + 36 * u**3 + 18 * u**2 + 6 * u + 1
    t = 6 * u**2 + 1
    assert bn.h * bn.r == bn.p + 1 - t
    for name in ("bls12_381", "bls12_377"):
        c = CURVES[name]
        u = c.u
        assert c.r == u**4 - u**2 + 1
        assert c.p == (u - 1) ** 2 * c.r // 3 + u
        assert ((u - 1) ** 2 * c.r) % 3 == 0
        t = u + 1
        assert c.h * c.r == c.p + 1 - t


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_generator_on_curve_and_order_r(c):
    assert ec.on_curve(c.G, c)
    assert ec.mul(c.r, c.G, c) is None
    assert ec.mul(c.r - 1, c.G, c) == ec.neg(c.G, c)


def test_mnt4_hasse_bound():
    # h = 1: #E = r must lie in the Hasse interval |p + 1 - #E| <= 2 sqrt(p)
    c = CURVES["mnt4_753"]
    t = c.p + 1 - c.r
    assert t * t <= 4 * c.p


def test_bn254_2G_published():
    g = json.load(open(os.path.join(GOLD, "known_points.json")))["bn254_2G"]
    c = CURVES["bn254"]
    assert ec.double(c.G, c) == (int(g["x"], 16), int(g["y"], 16))
