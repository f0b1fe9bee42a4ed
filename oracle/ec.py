"""Affine short-Weierstrass arithmetic for the oracle (test infrastructure only).

Points are (x, y) tuples of ints in [0, p); the point at infinity O is None.
PADD follows Formula (1):
    n = (y2 - y1) / (x2 - x1),  x3 = n^2 - x1 - x2,  y3 = n (x1 - x3) - y1
PDBL (the paper names it at PAPER.md:88 but prints no formula) is the textbook
tangent rule n = (3 x1^2 + a) / (2 y1), same x3, y3.  PMUL is left-to-right
double-and-add, "similar to the fast exponentiation technique".
"""
from .field import inv

O = None


def on_curve(P, c) -> bool:
    if P is None:
        return True
    x, y = P
    return 0 <= x < c.p and 0 <= y < c.p and (y * y - (x * x * x + c.a * x + c.b)) % c.p == 0


def neg(P, c):
    if P is None:
        return None
    return (P[0], (-P[1]) % c.p)


def double(P, c):
    if P is None:
        return None
    x1, y1 = P
    if y1 == 0:
        return None
    p = c.p
    n = (3 * x1 * x1 + c.a) * inv(2 * y1, p) % p
    x3 = (n * n - 2 * x1) % p
    y3 = (n * (x1 - x3) - y1) % p
    return (x3, y3)


def add(P, Q, c):
    """Formula (1) with the cases the formula leaves out (P or Q = O, P = ±Q)."""
    if P is None:
        return Q
    if Q is None:
        return P
    x1, y1 = P
    x2, y2 = Q
    p = c.p
    if x1 == x2:
        if (y1 + y2) % p == 0:
            return None
        return double(P, c)
    n = (y2 - y1) * inv(x2 - x1, p) % p
    x3 = (n * n - x1 - x2) % p
    y3 = (n * (x1 - x3) - y1) % p
    return (x3, y3)


def mul(k: int, P, c):
    """PMUL k*P by left-to-right double-and-add. k >= 0."""
    assert k >= 0
    R = None
    for bit in bin(k)[2:] if k else "":
        R = double(R, c)
        if bit == "1":
            R = add(R, P, c)
    return R


def to_output(P):
    """Output encoding (R4): canonical affine, O -> (0, 0)."""
    return (0, 0) if P is None else P
