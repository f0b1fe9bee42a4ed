#!/usr/bin/env python3
"""A/B timing of variant libraries: runs bench.py once per variants/libmsm_*.so (MSM_LIB)
and prints the stage times.  Usage: python tools/ab.py [--log2n 24] [--window-bits c] [names...]"""
import argparse
import glob
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ap = argparse.ArgumentParser()
ap.add_argument("--log2n", type=int, default=24)
ap.add_argument("--curve", default="bls12_381")
ap.add_argument("--window-bits", type=int, default=0)
ap.add_argument("--steps", type=int, default=3)
ap.add_argument("names", nargs="*")
a = ap.parse_args()
libs = sorted(glob.glob(os.path.join(ROOT, "variants", "libmsm_*.so")))
if a.names:
    libs = [l for l in libs if os.path.basename(l)[7:-3] in a.names]
for lib in libs:
    env = dict(os.environ, MSM_LIB=lib)
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--log2n", str(a.log2n), "--curve", a.curve, "--steps",
           str(a.steps), "--no-e2e", "--no-cpu-baseline", "--check"]
    if a.window_bits:
        cmd += ["--window-bits", str(a.window_bits)]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True)
    line = [l for l in r.stdout.splitlines() if l.startswith("{")]
    name = os.path.basename(lib)[7:-3]
    if not line:
        print(name, "FAILED", r.stderr[-500:])
        continue
    d = json.loads(line[-1])
    st = d["stages_ms"]
    print(json.dumps({"variant": name, "ms": round(d["ms_per_step"], 2), "acc_ms": st["accumulate_ms"],
                      "sort_ms": st["sort_ms"], "reduce_ms": st["reduce_ms"], "combine_ms": st["combine_ms"],
                      "frac": round(d["roofline"]["frac"], 4), "c": d["config"]["window_bits"],
                      "check": d.get("check")}), flush=True)
