"""Generated inputs for the oracle (test infrastructure only).

Points are P_i = e_i * G with e_i = e0 + i*delta mod r (DESIGN.md input recipe),
so that the closed form Q = (sum k_i e_i mod r) G applies.  (e0, delta) come from
the seeded generator `synth` (random numbers only, no curve arithmetic there).
P_0 = e0 G by double-and-add; P_{i+1} = P_i + D with D = delta G (Formula (1)).
"""
from . import ec


def progression_points(e0: int, delta: int, n: int, c):
    P = ec.mul(e0 % c.r, c.G, c)
    D = ec.mul(delta % c.r, c.G, c)
    out = []
    for _ in range(n):
        out.append(P)
        P = ec.add(P, D, c)
    return out


def progression_scalars(e0: int, delta: int, n: int, c):
    return [(e0 + i * delta) % c.r for i in range(n)]
