#!/usr/bin/env python3
"""Small-n driver for compute-sanitizer (memcheck / racecheck / synccheck): runs every
kernel of the library at n = 2^10 .. 2^14 on every curve — the three a3 sort variants, the
f3 table on and off, the f1 bucket split, logical multi-shard contexts, the pipelined API,
the debug field/EC/digit kernels — and checks each result against the oracle's closed form
(a sanitizer run must also be a correct run).

    compute-sanitizer --tool memcheck python tools/sanitize_driver.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402
from oracle import ec  # noqa: E402
from oracle.curves import CURVES  # noqa: E402
from paper_conf_asplos_ji0x024_b200 import msm  # noqa: E402

L32 = {"bn254": 8, "bls12_377": 12, "bls12_381": 12, "mnt4_753": 24}
S_W = {"bn254": 8, "bls12_377": 8, "bls12_381": 8, "mnt4_753": 24}


def main():
    import torch
    sizes = [int(a) for a in sys.argv[1:]] or [10, 12, 14]
    runs = 0
    for name in ("bn254", "bls12_377", "bls12_381", "mnt4_753"):
        c = CURVES[name]
        for lg in sizes:
            n = 1 << (lg if name != "mnt4_753" else min(lg, 12))
            e0, d = synth.point_seeds(c.r, lg)
            pts = torch.empty((n, 2 * L32[name]), dtype=torch.int32, device="cuda")
            msm.gen_points(name, e0, d, n, pts)
            ks = synth.scalars_range(c.r, 0, n, lg + 1)
            es = [(e0 + i * d) % c.r for i in range(n)]
            want = ec.to_output(ec.mul(sum(k * e for k, e in zip(synth.words_to_ints(ks), es)) % c.r, c.G, c))
            configs = [dict(pre=1), dict(pre=0, c=7), dict(pre=0, c=9, sort=1), dict(pre=1, c=8, sort=2),
                       dict(pre=0, c=6, sort=3), dict(pre=1, c=11, sort=3)]
            for cfg in configs:
                ctx = msm.Context(name, pts, n=n)
                ctx.set_option(msm.OPT_PRECOMPUTE, cfg["pre"])
                if "c" in cfg:
                    ctx.set_option(msm.OPT_WINDOW_BITS, cfg["c"])
                if "sort" in cfg:
                    ctx.set_option(msm.OPT_SORT, cfg["sort"])
                assert ctx.run(ks) == want, (name, n, cfg)
                runs += 1
                ctx.close()
            # f1 bucket split, 3 parts
            pw = msm.partial_words(name)
            parts = np.zeros(3 * pw, dtype=np.uint32)
            for g in range(3):
                ctx = msm.Context(name, pts, n=n)
                ctx.set_option(msm.OPT_SPLIT_PARTS, 3)
                ctx.set_option(msm.OPT_SPLIT_INDEX, g)
                ctx.run_partial(ks, parts[g * pw:(g + 1) * pw])
                ctx.close()
            assert msm.finalize(name, parts, 3) == want
            # logical shards + pipelined API
            ctx = msm.Context(name, pts, n=n, devices=[0, 0, 0])
            assert ctx.run(ks) == want
            ctx.close()
            ctx = msm.Context(name, pts, n=n)
            t0 = ctx.submit(ks)
            t1 = ctx.submit(ks)
            assert ctx.wait(t0) == want and ctx.wait(t1) == want
            ctx.close()
            runs += 3
        # debug kernels
        a = np.stack([synth.int_to_words(v % c.p, L32[name]) for v in range(1, 65)])
        for op in range(9):
            msm.debug_field(name, op, a, a[::-1].copy())
        msm.debug_digits(name, 5, synth.scalars(c.r, 64, 3))
        print(f"{name}: ok", flush=True)
    runs += round2_paths()
    print(f"sanitize driver: {runs} MSM runs, all equal to the closed form")


def round2_paths():
    """Round-2 kernels and host paths on BLS12-381: oversized sub-bins of the staged sort
    (k_s3_big_count / scan / big, equal scalars: ~10 buckets of n entries each), the
    two-pass cluster sort, chunked host-scalar upload with INIT accumulation, CUDA-graph
    replay of a device scalar buffer, and the small-n autotune (context creation)."""
    import torch
    name, lg = "bls12_381", 14
    c = CURVES[name]
    n = 1 << lg
    e0, d = synth.point_seeds(c.r, 99)
    pts = torch.empty((n, 2 * L32[name]), dtype=torch.int32, device="cuda")
    msm.gen_points(name, e0, d, n, pts)
    es = [(e0 + i * d) % c.r for i in range(n)]
    runs = 0
    for kind in ("equal", "uniform"):
        ks = synth.pattern_scalars(c.r, n, 98, kind) if kind == "equal" else synth.scalars_range(c.r, 0, n, 97)
        want = ec.to_output(ec.mul(sum(k * e for k, e in zip(synth.words_to_ints(ks), es)) % c.r, c.G, c))
        for cfg in (dict(sort=3, pre=0, c=6), dict(sort=4, pre=1, c=8), dict(sort=3, pre=1, c=10, chunks=3)):
            ctx = msm.Context(name, pts, n=n)  # n = 2^14: the creation autotune runs too
            ctx.set_option(msm.OPT_PRECOMPUTE, cfg["pre"])
            ctx.set_option(msm.OPT_WINDOW_BITS, cfg["c"])
            ctx.set_option(msm.OPT_SORT, cfg["sort"])
            if "chunks" in cfg:
                ctx.set_option(msm.OPT_H2D_CHUNKS, cfg["chunks"])
            assert ctx.run(ks) == want, (kind, cfg)
            runs += 1
            ctx.close()
        ctx = msm.Context(name, pts, n=n)
        kd = torch.from_numpy(ks.view(np.int32)).cuda()
        for _ in range(3):  # launch, capture, replay
            assert ctx.run(kd) == want, (kind, "graph")
            runs += 1
        ctx.close()
    print("round-2 paths: ok", flush=True)
    return runs


if __name__ == "__main__":
    main()
