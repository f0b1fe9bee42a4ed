#!/usr/bin/env python3
"""Build paper_conf_asplos_ji0x024_b200/libmsm.so (sm_100a) in-tree.

Each curve's kernels are a separate translation unit compiled in parallel; objects are
cached under build/ and rebuilt when any source or header is newer.  Usage:
    python tools/build.py [-j N] [--force]
"""
import argparse
import concurrent.futures as cf
import glob
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_asplos_ji0x024_b200")
CSRC = os.path.join(PKG, "csrc")
OUT = os.path.join(PKG, "libmsm.so")
BUILD = os.path.join(ROOT, "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-Xptxas", "-v", "-I", os.path.join(ROOT, "include")]


def newest_header():
    hs = glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + \
        glob.glob(os.path.join(ROOT, "include", "*.h"))
    return max(os.path.getmtime(h) for h in hs)


def compile_one(src, force, build_dir=BUILD, defines=()):
    obj = os.path.join(build_dir, os.path.basename(src).replace(".cu", ".o"))
    log = obj + ".log"
    if not force and os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(src), newest_header()):
        return obj, "cached"
    cmd = [NVCC] + FLAGS + [f"-D{d}" for d in defines] + ["-c", src, "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    with open(log, "w") as f:
        f.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr[-4000:]}")
    return obj, "built"


def build(jobs=8, force=False, verbose=True, only=None, defines=(), out=OUT, build_dir=BUILD, dev=None):
    """only: curve TU names to (re)compile (others reuse build_dir objects: dev/variants);
    defines: extra -D macros (kernel variants for A/B runs);
    dev: curve TU names to compile AND link (with engine.cu) -- a fast development library
    in which the other curves report MSM_ERR_CURVE (their factories are weak symbols)."""
    os.makedirs(build_dir, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    if dev:
        srcs = [s for s in srcs if "curve_" not in s or any(d in s for d in dev)]
        res = [compile_one(s, force, build_dir, defines) for s in srcs] if jobs == 1 else \
            list(cf.ThreadPoolExecutor(max_workers=jobs).map(lambda s: compile_one(s, force, build_dir, defines), srcs))
        objs = [o for o, _ in res]
        cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", out] + objs
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("link failed:\n" + r.stderr[-4000:])
        if verbose:
            print("built (dev: %s)" % ",".join(dev), out)
        return out
    if only:
        keep = [s for s in srcs if "curve_" not in s or any(o in s for o in only)]
        stale = [s for s in srcs if s not in keep]
        srcs = keep
        for s_ in stale:  # reuse objects from the main build dir
            o = os.path.join(build_dir, os.path.basename(s_).replace(".cu", ".o"))
            src_o = os.path.join(BUILD, os.path.basename(s_).replace(".cu", ".o"))
            if build_dir != BUILD and not os.path.exists(o):
                import shutil
                shutil.copy(src_o, o)
    # MNT4-753 is the slowest TU: start it first
    srcs.sort(key=lambda s: 0 if "mnt4" in s else 1)
    with cf.ThreadPoolExecutor(max_workers=jobs) as ex:
        res = list(ex.map(lambda s: compile_one(s, force, build_dir, defines), srcs))
    objs = sorted(glob.glob(os.path.join(build_dir, "*.o")))
    if verbose:
        for o, st in res:
            print(f"  {os.path.basename(o)}: {st}")
    if force or not os.path.exists(out) or any(os.path.getmtime(o) > os.path.getmtime(out) for o in objs):
        cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", out] + objs
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("link failed:\n" + r.stderr[-4000:])
    if verbose:
        print("built", out)
    return out


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("-j", type=int, default=8)
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--only", default="", help="comma-separated curve TUs to compile (dev)")
    ap.add_argument("-D", action="append", default=[], help="extra macro for a variant build")
    ap.add_argument("--out", default=OUT)
    ap.add_argument("--build-dir", default=BUILD)
    ap.add_argument("--dev", default="", help="comma-separated curve TUs: compile+link only these (fast dev lib)")
    a = ap.parse_args()
    try:
        build(a.j, a.force, only=[o for o in a.only.split(",") if o], defines=a.D, out=a.out, build_dir=a.build_dir,
              dev=[d for d in a.dev.split(",") if d] or None)
    except RuntimeError as e:
        print(e, file=sys.stderr)
        sys.exit(1)
