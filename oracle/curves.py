"""Curve constants for the oracle (test infrastructure only; see oracle/__init__.py).

PAPER.md Table 1 gives only the bit widths of k_i and P_i for
BN254 / BLS12-377 / BLS12-381 / MNT4753.  The constants themselves are the
standard published parameter sets (reading R1):
  BN254      alt_bn128 (EIP-196)
  BLS12-381  zkcrypto / IETF pairing-friendly-curves
  BLS12-377  Zexe / arkworks
  MNT4-753   Coda / Mina (arkworks ark-mnt4-753)
They are pinned in tests/test_oracle_constants.py against what the mathematics
fixes (primality, Table-1 bit widths, the curve-family closed forms in the seed
u, #E = h*r, G on the curve, r*G = O) — not against another copy of themselves.

Curve equation (short Weierstrass): y^2 = x^3 + a*x + b over F_p; G1 = the order-r
subgroup.  lam = bit length of r (the paper's λ).
"""
from dataclasses import dataclass


@dataclass(frozen=True)
class Curve:
    name: str
    p: int          # base-field prime
    r: int          # scalar-field prime (order of G1)
    a: int
    b: int
    gx: int         # generator of G1 (affine)
    gy: int
    h: int          # cofactor
    u: int | None   # family seed (None for MNT4-753)

    @property
    def lam(self) -> int:
        """λ: bit length of the scalars (Table 1 row k_i)."""
        return self.r.bit_length()

    @property
    def pbits(self) -> int:
        """Bit length of the base field (Table 1 row P_i)."""
        return self.p.bit_length()

    @property
    def L(self) -> int:
        """Number of 32-bit words of a base-field element."""
        return (self.pbits + 31) // 32

    @property
    def S(self) -> int:
        """Number of 32-bit words of a scalar."""
        return (self.lam + 31) // 32

    @property
    def G(self):
        return (self.gx, self.gy)


BN254 = Curve(
    name="bn254",
    p=0x30644e72e131a029b85045b68181585d97816a916871ca8d3c208c16d87cfd47,
    r=0x30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001,
    a=0, b=3, gx=1, gy=2, h=1,
    u=0x44e992b44a6909f1,
)

BLS12_381 = Curve(
    name="bls12_381",
    p=0x1a0111ea397fe69a4b1ba7b6434bacd764774b84f38512bf6730d2a0f6b0f6241eabfffeb153ffffb9feffffffffaaab,
    r=0x73eda753299d7d483339d80809a1d80553bda402fffe5bfeffffffff00000001,
    a=0, b=4,
    gx=0x17f1d3a73197d7942695638c4fa9ac0fc3688c4f9774b905a14e3a3f171bac586c55e83ff97a1aeffb3af00adb22c6bb,
    gy=0x08b3f481e3aaa0f1a09e30ed741d8ae4fcf5e095d5d00af600db18cb2c04b3edd03cc744a2888ae40caa232946c5e7e1,
    h=0x396c8c005555e1568c00aaab0000aaab,
    u=-0xd201000000010000,
)

BLS12_377 = Curve(
    name="bls12_377",
    p=0x1ae3a4617c510eac63b05c06ca1493b1a22d9f300f5138f1ef3622fba094800170b5d44300000008508c00000000001,
    r=0x12ab655e9a2ca55660b44d1e5c37b00159aa76fed00000010a11800000000001,
    a=0, b=1,
    gx=0x08848defe740a67c8fc6225bf87ff5485951e2caa9d41bb188282c8bd37cb5cd5481512ffcd394eeab9b16eb21be9ef,
    gy=0x01914a69c5102eff1f674f5d30afeec4bd7fb348ca3e52d96d182ad44fb82305c2fe3d3634a9591afd82de55559c8ea6,
    h=0x170b5d44300000000000000000000000,
    u=0x8508c00000000001,
)

MNT4_753 = Curve(
    name="mnt4_753",
    p=0x01c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db117e776f218059db80f0da5cb537e38685acce9767254a4638810719ac425f0e39d54522cdd119f5e9063de245e8001,
    r=0x01c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db26c5c28c859a99b3eebca9429212636b9dff97634993aa4d6c381bc3f0057974ea099170fa13a4fd90776e240000001,
    a=2,
    b=0x01373684a8c9dcae7a016ac5d7748d3313cd8e39051c596560835df0c9e50a5b59b882a92c78dc537e51a16703ec9855c77fc3d8bb21c8d68bb8cfb9db4b8c8fba773111c36c8b1b4e8f1ece940ef9eaad265458e06372009c9a0491678ef4,
    gx=0x0542f1dad450bb76a02d86daaffbaeb69995eb9efa5546444d40c82d6a271f1a438626d1ef781d1de4ffb1f806b314c5ad3463d98a4ea009d57aad9716f708885feff338dd73a5a7eeecfbce7cf95d3c2ab23be1c24740af0fdeb3b7f1981,
    gy=0x04ab6473526e257b175ae94deb9e10aba4ba72f7fddcdea19cb10b2bf61f37ae2c456ee5599dd7c3dfa4100284833115aec5dea57ef53ee29157bdf1b741aebd423036db8fb990a342449caeb92fa6b031ea99cff05e05ec3be2e4a050358,
    h=1,
    u=None,
)

CURVES = {c.name: c for c in (BN254, BLS12_377, BLS12_381, MNT4_753)}
