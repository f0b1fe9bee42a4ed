"""CPU oracle for the MSM hot path — TEST INFRASTRUCTURE ONLY.

This package is the plain, slow, obviously-correct reference for what the CUDA
path computes: Q = sum_i k_i * P_i over G1 of BN254, BLS12-377, BLS12-381 and
MNT4-753 (§2.2).  It is written in pure Python integers, follows
the paper's formulas in the paper's notation, and shares no code, constants or
helpers with the product package `paper_conf_asplos_ji0x024_b200` (neither
imports the other).

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` /
`--impl reference` legs may import anything from here.  The product path must
never route through this package.

Modules
-------
curves    curve constants (Table 1 gives only bit widths; the values are
          the standard published parameter sets, pinned in tests/test_oracle_*)
field     modular arithmetic and Montgomery multiplication, SOS (Alg. 2)
ec        affine point arithmetic, Formula (1) + tangent doubling
xyzz      XYZZ PADD (Alg. 1), PACC (Alg. 4), PDBL
msm       three independent MSM routes: naive, plain Pippenger,
          closed form for generated inputs
stages    the staged decomposition the GPU uses (signed digits, buckets,
          bucket-reduce, window-reduce) for stage-level parity
points    generated inputs P_i = e_i * G
"""
