#!/usr/bin/env python3
"""bench.py — MSM latency / throughput of the B200 library on BASELINE.json's headline
workload (default: BLS12-381 G1, n = 2^26, config C4), one JSON line on rank 0.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--curve C] [--log2n L] [--impl reference]

N = 1: one process, one context on cuda:0.  N > 1 (launched by torchrun, one process per
GPU, NCCL): the n points are split into N contiguous shards (strong scaling: total n fixed);
each rank computes its partial MSM (msm_run_partial), the partials are all-gathered over
NCCL and rank 0 adds them (msm_finalize).  A "step" is one whole MSM of n points.

Timing: W untimed warm-ups; K timed steps between a barrier + cuda.synchronize on both
sides; CUDA events on the library's stream; max over ranks.  The inputs (points 112 B x n,
scalars 32 B x n) exceed the 126 MB L2 many times, so no explicit flush is needed.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CURVE_INFO = {  # name: (L32, S, lambda, L (radix-2^W limbs), W)
    "bn254": (8, 8, 254, 9, 30),
    "bls12_377": (12, 8, 253, 13, 30),
    "bls12_381": (12, 8, 255, 13, 30),
    "mnt4_753": (24, 24, 753, 27, 29),
}
METRIC = "MSM latency (ms) and points/sec at 2^20–2^26, 1/2/4/8 B200; % IMAD roofline"
PAPER_MS = {("bls12_381", 26, 1): 855.2, ("bls12_381", 26, 8): 113.7, ("bls12_377", 24, 1): 213.6,
            ("bls12_377", 24, 8): 30.35, ("mnt4_753", 22, 1): 863.8, ("mnt4_753", 22, 8): 116.8}


def imad_slots_per_mult(L):
    """IMAD-pipe issue slots of one radix-2^W Montgomery multiplication as implemented:
    2L^2 limb products as IMAD.WIDE.U32 (2 slots each on sm_100a: half rate, measured in
    microbench/imad_peak.cu) + L low-only IMAD for m_k = t_k n'_0 (1 slot)."""
    return 2 * L * L * 2 + L


def imad_slots_per_sqr(L):
    """Squaring: L(L+1)/2 a*a products + L^2 m*p products (2 slots each) + L m_k."""
    return 2 * (L * (L + 1) // 2 + L * L) + L


def imad_slots_per_sum(L):
    """fmul_sum (a*b + c*d under one Montgomery reduction): 3 L^2 products (2 slots) + L m_k."""
    return 3 * L * L * 2 + L


def imad_slots_per_pacc(L):
    """PACC (Alg. 4) as implemented: 6 multiplications + 2 squarings + one fmul_sum
    (Y' = R*D - Y*PPP with one reduction, ec.cuh MSM_ACC_SUM)."""
    return 6 * imad_slots_per_mult(L) + 2 * imad_slots_per_sqr(L) + imad_slots_per_sum(L)


def peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        return json.load(open(path))
    except Exception:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0, "fallback": True}


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.FIELDS,
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=5)
                if out.returncode == 0 and out.stdout.strip():
                    self.rows.append([v.strip() for v in out.stdout.strip().split(",")])
            except Exception:
                pass
            self._stop.wait(0.2)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 4 + i and r[4 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows),
                "power_w_max": max((float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()), default=None)}


def ncu_traffic(curve, log2n):
    """dram__bytes_read.sum + dram__bytes_write.sum of one k_accumulate launch, from the
    committed ncu --set full capture of this workload (profiles/ncu_traffic.json), or None."""
    try:
        t = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))[f"{curve} 2^{log2n}"]
        return {"bytes": t["read"] + t["write"], "read": t["read"], "write": t["write"],
                "algorithmic_bytes": t.get("algorithmic"), "source": t["source"]}
    except Exception:
        return None


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ---------------------------------------------------------------------------------------
# CPU baseline: the oracle's plain Pippenger, as it
# stands, on every host core: worker w owns points [w*chunk, (w+1)*chunk) of a prefix of
# the bench workload (same curve, same input recipe), computes the MSM of its chunk, and
# the partial points are summed.  The timed region is the Pippenger only (input generation
# happens before a barrier).  The rate (points/s) is extrapolated to the full n, labelled.
ORACLE_S = {"bn254": 8, "bls12_377": 8, "bls12_381": 8, "mnt4_753": 8}
ORACLE_CHUNK = {"bn254": 1 << 13, "bls12_377": 1 << 13, "bls12_381": 1 << 13, "mnt4_753": 1 << 9}


def _oracle_worker(curve, seed, off, cnt, s, barrier, conn):
    sys.path.insert(0, ROOT)
    import synth
    from oracle import points as opoints
    from oracle import msm as omsm
    from oracle.curves import CURVES
    c = CURVES[curve]
    e0, d = synth.point_seeds(c.r, seed)
    Ps = opoints.progression_points(synth.progression_offset(c.r, e0, d, off), d, cnt, c)
    ks = synth.words_to_ints(synth.scalars_range(c.r, off, cnt, seed))
    while True:
        cmd = conn.recv()
        if cmd != "run":
            break
        barrier.wait()
        t0 = time.perf_counter()
        Q = omsm.msm_pippenger(ks, Ps, c, s=s)
        t1 = time.perf_counter()
        conn.send((t0, t1, Q))


def cpu_info():
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    if model is None:
        try:
            for line in open("/proc/cpuinfo"):
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
        except Exception:
            pass
    try:
        cores = len(os.sched_getaffinity(0))
    except Exception:
        cores = os.cpu_count() or 1
    return cores, model


class OraclePool:
    """One spawned process per host core, each holding its chunk of the sample."""

    def __init__(self, curve, seed, workers=None, chunk=None):
        import multiprocessing as mp
        cores, self.model = cpu_info()
        self.workers = workers or cores
        self.chunk = chunk or ORACLE_CHUNK[curve]
        self.s = ORACLE_S[curve]
        self.curve = curve
        self.n_sample = self.workers * self.chunk
        ctx = mp.get_context("spawn")
        self.barrier = ctx.Barrier(self.workers)
        self.conns, self.procs = [], []
        for w in range(self.workers):
            a, b = ctx.Pipe()
            p = ctx.Process(target=_oracle_worker, args=(curve, seed, w * self.chunk, self.chunk, self.s, self.barrier, b),
                            daemon=True)
            p.start()
            self.conns.append(a)
            self.procs.append(p)

    def run(self):
        """(wall seconds of the parallel Pippenger, Q = sum of the chunk MSMs)."""
        sys.path.insert(0, ROOT)
        from oracle import ec
        from oracle.curves import CURVES
        for cn in self.conns:
            cn.send("run")
        res = [cn.recv() for cn in self.conns]
        wall = max(r[1] for r in res) - min(r[0] for r in res)
        c = CURVES[self.curve]
        Q = None
        for r in res:
            Q = ec.add(Q, r[2], c)
        return wall, Q

    def close(self):
        for cn in self.conns:
            try:
                cn.send("stop")
            except Exception:
                pass
        for p in self.procs:
            p.join(timeout=5)
            if p.is_alive():
                p.terminate()

    def describe(self, wall, n_full):
        return (f"{self.curve}: {self.n_sample}-point prefix of the n={n_full} workload "
                f"({self.workers} processes x {self.chunk} points, oracle.msm_pippenger s={self.s}, pure-Python ints, "
                f"partials summed); {wall:.2f} s wall; points/s extrapolated linearly to n (Pippenger cost per point "
                f"is ~constant in n at fixed s)")


def cpu_baseline(curve, n_full, seed):
    """SURVEY.md §8(d) CPU baseline, one bounded run on all host cores."""
    pool = OraclePool(curve, seed)
    try:
        wall, _ = pool.run()
    finally:
        pool.close()
    return {"value": pool.n_sample / wall, "unit": "points/s", "cores": pool.workers, "cpu_model": pool.model,
            "kind": "oracle", "sample": pool.describe(wall, n_full), "seconds": wall,
            "extrapolated_ms_full_n": n_full / (pool.n_sample / wall) * 1e3}


def run_reference(args):
    """Reference arm (tier framing): the oracle as it stands on the host cores, each step a
    bounded sample of the bench workload.  Rank 0 only; other ranks exit at once."""
    ws, rank, local = dist_env()
    if rank != 0:
        return 0
    curve = args.curve
    seed = 20240427 + 3
    cores, _ = cpu_info()
    chunk = args.ref_sample // cores if args.ref_sample else max(64, ORACLE_CHUNK[curve] // 8)
    pool = OraclePool(curve, seed, chunk=chunk)
    try:
        for _ in range(args.warmup):
            pool.run()
        times = [pool.run()[0] for _ in range(args.steps)]
    finally:
        pool.close()
    ms = statistics.median(times) * 1e3
    val = pool.n_sample / (ms / 1e3)
    n = 1 << args.log2n
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": "points/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int (python big ints)", "data": "synthetic",
        "config": {"workload": f"{curve} G1 MSM n=2^{args.log2n}", "curve": curve, "n": n,
                   "sample_n": pool.n_sample, "l2": "n/a (CPU)"},
        "cpu_baseline": {"value": val, "unit": "points/s", "cores": pool.workers, "cpu_model": pool.model,
                         "kind": "oracle", "sample": pool.describe(ms / 1e3, n)},
        "e2e": {"value": val, "unit": "points/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def self_launch(args):
    """`python bench.py --gpus N` outside torchrun: re-run this script under
    torch.distributed.run with N ranks (one process per GPU, 127.0.0.1 rendezvous)."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.run(cmd).returncode


# ---------------------------------------------------------------------------------------
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--curve", default="bls12_381", choices=list(CURVE_INFO))
    ap.add_argument("--log2n", type=int, default=26)
    ap.add_argument("--window-bits", type=int, default=0)
    ap.add_argument("--precompute", type=int, default=2, choices=[0, 1, 2],
                    help="f3 window table (PAPER.md:147): 0 off, 1 on, 2 auto (library default)")
    ap.add_argument("--sort", type=int, default=0, choices=[0, 1, 2, 3, 4],
                    help="a3 variant (MSM_OPT_SORT): 0 auto, 1 direct global atomics (ablation), 2 binned, "
                         "3 three-level staged, 4 two-pass cluster")
    ap.add_argument("--split", default="auto", choices=["auto", "points", "buckets"],
                    help="N > 1 decomposition: point shards, or the paper's bucket split (PAPER.md:223); "
                         "auto = buckets for N > 1")
    ap.add_argument("--acc-mode", type=int, default=2, choices=[0, 1, 2],
                    help="a4 (MSM_OPT_ACC_MODE): 0 PACC only, 1 batch-affine front end + PACC, 2 auto (library default)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-sample", type=int, default=0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-check", action="store_true",
                    help="skip the closed-form check of the result (run by default after the timed region)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return self_launch(args)

    import numpy as np
    import torch

    import synth
    from paper_conf_asplos_ji0x024_b200 import msm
    from paper_conf_asplos_ji0x024_b200.dist import gather_and_finalize, shard_bounds

    ws, rank, local = dist_env()
    if ws != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE {ws}; using WORLD_SIZE", file=sys.stderr)
    # Shared-device mode (test only; automatic when the box has fewer GPUs than ranks, or
    # MSM_BENCH_SHARE_DEVICE=1): every rank on cuda:0 and the gather over gloo with host
    # partials, so the N > 1 path runs end to end on a one-GPU box.  Its timings are not
    # scaling numbers (the ranks share one GPU) and the line says so.
    share = os.environ.get("MSM_BENCH_SHARE_DEVICE") == "1" or (ws > 1 and torch.cuda.device_count() < ws)
    if share and ws > 1 and rank == 0:
        print(f"bench.py: shared-device mode ({ws} ranks on cuda:0, gloo gather)", file=sys.stderr)
    torch.cuda.set_device(0 if share else local)
    dev = torch.device("cuda", 0 if share else local)
    coll_dev = torch.device("cpu") if share else dev
    if ws > 1:
        import torch.distributed as dist
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    curve = args.curve
    L32, S, lam, L, W = CURVE_INFO[curve]
    r = synth.CURVE_ORDERS[curve]
    n = 1 << args.log2n
    # multi-GPU decomposition: "points" = contiguous point shards (north_star), "buckets" =
    # the paper's bucket split (f1): every rank holds all n points and scalars
    # and sums the buckets |d| = ws*q + rank of every bucket set
    split = args.split if args.split != "auto" else ("buckets" if ws > 1 and not share else "points")
    off, n_g = shard_bounds(n, ws, rank) if split == "points" else (0, n)
    seed = 20240427 + 3
    e0, delta = synth.point_seeds(r, seed)

    # inputs: points generated on the device by the library's generator (not timed),
    # scalars drawn on the host (numpy PCG64) and uploaded once for the HBM-resident runs.
    t0 = time.time()
    pts = torch.empty((n_g, 2 * L32), dtype=torch.int32, device=dev)
    msm.gen_points(curve, synth.progression_offset(r, e0, delta, off), delta, n_g, pts)
    ks_host = synth.scalars_range(r, off, n_g, seed)
    ks_pinned = torch.from_numpy(ks_host.view(np.int32)).pin_memory()
    ks_dev = ks_pinned.to(dev, non_blocking=False)
    if share and ws > 1:
        # ranks sharing one GPU create their contexts (and f3 tables) one after another, so
        # each planner sees the memory the previous ones took
        for turn in range(ws):
            if turn == rank:
                ctx = msm.Context(curve, pts, ngpus=1, n=n_g)
            torch.distributed.barrier()
    else:
        ctx = msm.Context(curve, pts, ngpus=1, n=n_g)
    assert ctx.get_option(msm.OPT_DEVICE) == dev.index, "context not on this rank's device"
    del pts
    torch.cuda.empty_cache()
    if args.precompute != 2:
        ctx.set_option(msm.OPT_PRECOMPUTE, args.precompute)
    if args.window_bits:
        ctx.set_option(msm.OPT_WINDOW_BITS, args.window_bits)
    if args.sort:
        ctx.set_option(msm.OPT_SORT, args.sort)
    if args.acc_mode != 2:
        ctx.set_option(msm.OPT_ACC_MODE, args.acc_mode)
    if split == "buckets" and ws > 1:
        ctx.set_option(msm.OPT_SPLIT_PARTS, ws)
        ctx.set_option(msm.OPT_SPLIT_INDEX, rank)
    setup_s = time.time() - t0
    stream = torch.cuda.ExternalStream(ctx.stream(0), device=dev)
    pw = msm.partial_words(curve)
    partial = torch.zeros(pw, dtype=torch.int32, device=coll_dev)

    def step(scalars):
        if ws == 1:
            return ctx.run_words(scalars)
        ctx.run_partial(scalars, partial)          # a2..a6 on this rank's shard
        return gather_and_finalize(curve, partial)  # a7: NCCL all-gather + msm_finalize on rank 0

    def barrier():
        torch.cuda.synchronize()
        if ws > 1:
            torch.distributed.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        step(ks_dev)
    barrier()
    # timed: HBM-resident scalars
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    acc_ms, stage = [], []
    sampler = ClockSampler(local)
    with sampler:
        barrier()
        for i in range(args.steps):
            ev[i][0].record(stream)
            res = step(ks_dev)
            ev[i][1].record(stream)
            st = ctx.stats()
            acc_ms.append(st["accumulate_ms"])
            stage.append(st)
        barrier()
    graph_note = ""
    if stage and stage[-1]["accumulate_ms"] < 0:
        # small n: the timed steps replayed a CUDA graph (MSM_OPT_GRAPH), which has no
        # per-stage events; the roofline's kernel time comes from 3 un-graphed steps
        ctx.set_option(msm.OPT_GRAPH, 0)
        acc_ms, stage = [], []
        for _ in range(3):
            step(ks_dev)
            st = ctx.stats()
            acc_ms.append(st["accumulate_ms"])
            stage.append(st)
        ctx.set_option(msm.OPT_GRAPH, 1)
        graph_note = " (timed steps replayed a CUDA graph; stage times from 3 un-graphed steps after them)"
    times = [a.elapsed_time(b) for a, b in ev]
    my_ms = sum(times) / len(times)
    t_all = torch.tensor([my_ms], dtype=torch.float64, device=coll_dev)
    if ws > 1:
        torch.distributed.all_reduce(t_all, op=torch.distributed.ReduceOp.MAX)
    ms = float(t_all.item())

    # e2e: host (pinned) scalars through the same C-ABI call, H2D inside the timed region
    e2e = None
    if not args.no_e2e and ws == 1:
        # pipelined public API (msm_submit / msm_wait): every MSM copies its own scalars from
        # pinned host memory and reads back its result; MSM t+1's H2D overlaps MSM t
        ks_np = ks_pinned.numpy()
        ctx.wait_words(ctx.submit(ks_np))
        torch.cuda.synchronize()
        nst = max(2, min(args.steps, 5))
        t0 = time.perf_counter()
        pending, outs = [], []
        for i in range(nst):
            pending.append(ctx.submit(ks_np))
            if len(pending) == 2:
                outs.append(ctx.wait_words(pending.pop(0)))
        while pending:
            outs.append(ctx.wait_words(pending.pop(0)))
        e2e_ms = (time.perf_counter() - t0) * 1e3 / nst
        # every pipelined result equals the device-resident run's (same scalars)
        e2e_same = all(np.array_equal(np.asarray(o), np.asarray(res)) for o in outs)
        e2e = {"value": n / (e2e_ms / 1e3), "unit": "points/s", "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": n * S * 4, "d2h_bytes_per_step": 2 * L32 * 4,
               "timing": f"host wall clock around {nst} pipelined msm_submit/msm_wait calls (pinned host scalars, "
                         "each MSM's H2D overlaps the previous MSM's accumulation; the first one, submitted into an "
                         "empty pipeline, uploads in chunks), per MSM",
               "results_equal_device_run": bool(e2e_same)}
        # single-call latency (one msm_run per MSM, pinned host scalars, H2D inside): the
        # library default uploads the scalars in growing chunks, each sorted and accumulated
        # while the next one uploads (MSM_OPT_H2D_CHUNKS); one copy before the MSM for contrast
        single = {}
        for K, key in ((0, "chunked"), (1, "one_copy")):
            ctx.set_option(msm.OPT_H2D_CHUNKS, K)
            ctx.run_words(ks_np)
            ts = []
            for _ in range(3):
                s0 = time.perf_counter()
                ctx.run_words(ks_np)
                ts.append((time.perf_counter() - s0) * 1e3)
            single[key] = {"ms": sorted(ts)[1], "chunks": int(ctx.get_option(msm.OPT_H2D_CHUNKS))}
        ctx.set_option(msm.OPT_H2D_CHUNKS, 0)
        e2e["single_call"] = dict(single, timing="host wall clock around msm_run (median of 3)")
    elif not args.no_e2e:
        for _ in range(1):
            step(ks_pinned)
        barrier()
        t0 = time.perf_counter()
        e_ms = []
        for i in range(max(2, min(args.steps, 5))):
            s0 = time.perf_counter()
            step(ks_pinned.numpy() if ws == 1 else ks_pinned)
            if ws > 1:
                barrier()
            e_ms.append((time.perf_counter() - s0) * 1e3)
        e_t = torch.tensor([sum(e_ms) / len(e_ms)], dtype=torch.float64, device=coll_dev)
        if ws > 1:
            torch.distributed.all_reduce(e_t, op=torch.distributed.ReduceOp.MAX)
        e2e_ms = float(e_t.item())
        e2e = {"value": n / (e2e_ms / 1e3), "unit": "points/s", "ms_per_step": e2e_ms,
               "h2d_bytes_per_step": (n if split == "points" else n * ws) * S * 4, "d2h_bytes_per_step": 2 * L32 * 4,
               "timing": "host wall clock around msm_run with pinned host scalars (max over ranks)"}

    check = None
    if not args.no_check and rank == 0:
        t_chk = time.time()
        check = verify(curve, n, e0, delta, seed, ctx if ws == 1 else None, ks_dev, res, msm)
        check["seconds"] = round(time.time() - t_chk, 1)
        check["what"] = ("last timed step's affine result vs the oracle closed form (e0*sum k_i + delta*sum i*k_i "
                         "mod r)*G over all n scalars (oracle/msm.py closed_form_arith)")

    if rank != 0:
        ctx.close()
        if ws > 1:
            torch.distributed.barrier()
            torch.distributed.destroy_process_group()
        return 0

    # roofline of the dominant kernel (k_accumulate): algorithmic work =
    # PACC x 10 field mults x (4 L32^2 + L32) IMAD (CIOS on 32-bit limbs, L32 = 8/12/12/24)
    # per launch, over the kernel's CUDA-event time, against 148 SM x 64 IMAD/clk x max clock.
    # frac_pipe is the IMAD-pipe occupancy of the instruction stream actually run
    # (radix-2^W limbs: 2 slots per IMAD.WIDE), which is what ncu's fmaheavy counter sees.
    st = stage[-1]
    nonempty = ctx.get_option(msm.OPT_NONEMPTY)
    pacc = int(st["entries"]) - int(nonempty)
    imad_alg = pacc * 10 * (4 * L32 * L32 + L32)
    slots = pacc * imad_slots_per_pacc(L)
    acc_avg_ms = sum(acc_ms) / len(acc_ms)
    pk = peaks()
    sm_max = pk.get("sm_max_mhz", 1965.0)
    peak_imad = 148 * 64 * sm_max * 1e6
    achieved = imad_alg / (acc_avg_ms / 1e3)
    achieved_slots = slots / (acc_avg_ms / 1e3)
    # a3 (digits + counting sort) against HBM: algorithmic bytes = scalars read once
    # (n*S*4) + sorted entries written once (M*4); sort_ms is the stage's CUDA-event time on
    # the library stream
    sort_ms = sum(x["sort_ms"] for x in stage) / len(stage)
    sort_bytes = n_g * S * 4 + int(st["entries"]) * 4
    hbm_peak = pk.get("hbm_gbs", 6550.0)
    sort_gbs = sort_bytes / (sort_ms / 1e3) / 1e9 if sort_ms > 0 else None
    clocks = sampler.summary()
    cpu = None
    if not args.no_cpu_baseline and ws == 1:
        cpu = cpu_baseline(curve, n, seed)
    paper = PAPER_MS.get((curve, args.log2n, ws))
    line = {
        "metric": METRIC,
        "value": n / (ms / 1e3),
        "unit": "points/s",
        "n_gpus": ws,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": ms,
        "higher_is_better": True,
        "scaling": "strong",
        "vs_baseline": None,
        "dtype": "u32 (exact modular integer arithmetic, radix-2^%d limbs)" % W,
        "data": "synthetic: P_i = (e0 + i*delta) G generated on device, k_i uniform on [0, r) (numpy PCG64)",
        "config": {"workload": f"{curve} G1 MSM n=2^{args.log2n} (BASELINE.json config C4)" if (curve, args.log2n) == ("bls12_381", 26)
                   else f"{curve} G1 MSM n=2^{args.log2n}",
                   "curve": curve, "n": n, "window_bits": st["window_bits"], "nwin": st["nwin"],
                   "precompute": bool(st["precompute"]), "sort_variant": ctx.get_option(msm.OPT_SORT),
                   "bucket_sets": 1 if st["precompute"] else st["nwin"],
                   "parallelism": (f"point-sharded x{ws}" if split == "points" else f"bucket-split x{ws} (PAPER.md:223)")
                                  + ((" + gloo all-gather of host partials (shared-device test mode: all ranks on cuda:0, "
                                      "times are NOT scaling numbers)" if share else " + NCCL all-gather of partials")
                                     if ws > 1 else ""),
                   "shared_device": bool(share and ws > 1),
                   "scalars": "device-resident (HBM) for value; pinned host for e2e",
                   "l2": "inputs >> L2 (points %.1f GB + scalars %.1f GB per step); no flush needed" % (
                       n * (2 * L + 2) * 4 / 1e9, n * S * 4 / 1e9)},
        "roofline_sort": {"stage": "a3 digits + counting sort (all kernels between EV_H2D and EV_SORT)", "bound": "hbm",
                          "achieved": sort_gbs, "peak": hbm_peak, "unit": "GB/s",
                          "frac": (sort_gbs / hbm_peak) if sort_gbs else None, "traffic": None,
                          "work": f"{n_g} x {S * 4} B scalars + {int(st['entries'])} x 4 B sorted entries per step",
                          "peak_basis": "MEASURED_PEAKS.json hbm_gbs (copy bandwidth)"},
        "stages_ms": {k: round(v, 3) for k, v in st.items() if k.endswith("_ms") and k != "table_ms"},
        "latency_ms": {"mean": ms, "min": min(times), "max": max(times)},
        "roofline": {"kernel": "k_accumulate_sync", "bound": "alu",
                     "achieved": achieved / 1e12, "peak": peak_imad / 1e12, "unit": "T IMAD/s",
                     "frac": achieved / peak_imad, "traffic": ncu_traffic(curve, args.log2n),
                     "work": f"{pacc} PACC x 10 field mults x (4*{L32}^2+{L32} = {4 * L32 * L32 + L32}) IMAD "
                             f"(SURVEY.md §8(d): CIOS on 32-bit limbs) per launch",
                     "time_basis": f"k_accumulate CUDA-event average over the {args.steps} timed steps, library stream"
                                   + graph_note,
                     "peak_basis": f"148 SM x 64 IMAD/clk x {sm_max} MHz (clocks.max.sm; B200 guide unit counts)",
                     "frac_pipe": achieved_slots / peak_imad,
                     "frac_pipe_basis": f"IMAD-pipe slots of the radix-2^{W} instruction stream run: {pacc} PACC x "
                                        f"{imad_slots_per_pacc(L)} slots ("
                                        + f"6 mul x {imad_slots_per_mult(L)} + 2 sqr x {imad_slots_per_sqr(L)} + 1 fmul_sum x "
                                          f"{imad_slots_per_sum(L)}"
                                        + "), IMAD.WIDE = 2 slots (measured)",
                     "field_mults_per_s": pacc * 10 / (acc_avg_ms / 1e3)},
        "clocks": clocks,
        "gpu_launches": int(st["acc_launches"]) * args.steps + (args.steps if ws > 1 else 0),
        "setup_s": round(setup_s, 2),
        "table_build_s": round(st["table_ms"] / 1e3, 3) if st["precompute"] else 0.0,
    }
    if paper:
        line["paper_context"] = {"ms": paper, "hardware": f"{ws}x A100 80GB (DistMSM, PAPER.md Table 3)"}
    if e2e:
        line["e2e"] = e2e
    if cpu:
        line["cpu_baseline"] = cpu
    if check is not None:
        line["check"] = check
    print(json.dumps(line), flush=True)
    ctx.close()
    if ws > 1:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()
    return 0


def verify(curve, n, e0, delta, seed, ctx, ks_dev, res, msm):
    """Closed-form check (oracle): Q = (e0 * sum k_i + delta * sum i k_i mod r) G."""
    import numpy as np
    import synth
    from oracle import ec, msm as omsm
    from oracle.curves import CURVES
    c = CURVES[curve]
    ks = synth.scalars_range(c.r, 0, n, seed)
    S = ks.shape[1]
    sk, sik = 0, 0
    idx = np.arange(n, dtype=np.uint64)
    for w in range(S):
        col = ks[:, w].astype(np.uint64)
        sk += int(col.sum()) << (32 * w)
        for h in range(2):  # 16-bit halves keep i * half < 2^42, chunk sums < 2^62
            half = (col >> np.uint64(16 * h)) & np.uint64(0xFFFF)
            tot = 0
            for a in range(0, n, 1 << 20):
                tot += int((idx[a:a + (1 << 20)] * half[a:a + (1 << 20)]).sum())
            sik += tot << (32 * w + 16 * h)
    want = ec.to_output(omsm.closed_form_arith(sk, sik, e0, delta, c))
    got = res if isinstance(res, tuple) else msm.point_from_words(res, msm.field_words(curve))
    return {"closed_form_match": got == want}


if __name__ == "__main__":
    sys.exit(main())
