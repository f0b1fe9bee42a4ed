"""Multi-shard paths on the GPU, through the C-ABI.

* In-library sharding (ngpus > 1 in one process): per-shard pipelines, the gather of the G
  partial XYZZ points onto shard 0's device (peer / same-device copies; PAPER.md:163
  "only N_gpu points are left to sum") and the final add.  On a one-GPU box the shards are
  *logical* (msm_context_create_on with a repeated device): same code path, same-device
  copies.  Bit-exact against the oracle's closed form for G in {2, 4, 8} and
  n in {0, 1, G-1, 1000, 2^16}.
* Device binding: a context lands on the caller's current device (not device 0) and the
  caller's current device is unchanged by every call.
* Ordering: device scalars written by torch on its default stream immediately before the
  call are read after that write.
* The headline regime (ROADMAP: VERDICT r01 item 2): BLS12-381 at n = 2^20 with every
  default — automatic c, the f3 table, the staged three-level sort reached automatically
  (>= 2^21 entries), lockstep accumulation — bit-exact.
* `python bench.py --gpus 2` (self-launched torchrun; shared-device mode on a one-GPU box)
  exits 0 and its JSON line carries a passing closed-form check.
"""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import synth
from oracle import ec, msm as omsm
from oracle.curves import CURVES
from tests.helpers import L32, S_W, points_to_words, progression

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_asplos_ji0x024_b200 import msm as m
    assert m.device_count() >= 1, "no CUDA device"
    return m


def closed(name, ks, es):
    return ec.to_output(omsm.msm_closed_form(ks, es, CURVES[name]))


def gen_device_points(lib, name, n, seed):
    import torch
    c = CURVES[name]
    e0, d = synth.point_seeds(c.r, seed)
    pts = torch.empty((max(n, 1), 2 * L32[name]), dtype=torch.int32, device="cuda")
    if n:
        lib.gen_points(name, e0, d, n, pts)
    es = [(e0 + i * d) % c.r for i in range(n)]
    return pts, es


@pytest.mark.parametrize("name", ["bn254", "bls12_381", "mnt4_753"])
@pytest.mark.parametrize("G", [2, 4, 8])
def test_logical_shards_small(lib, name, G):
    c = CURVES[name]
    sizes = [0, 1, G - 1, 1000 if name != "mnt4_753" else 130]
    for n in sizes:
        Ps, es, _, _ = progression(name, max(n, 1), 51)
        Ps, es = list(Ps)[:n], list(es)[:n]
        ks = synth.words_to_ints(synth.scalars(c.r, n, 52 + n)) if n else []
        ctx = lib.Context(name, points_to_words(Ps, name), n=n, devices=[0] * G)
        try:
            assert ctx.get_option(lib.OPT_NGPUS) == G
            offs = [ctx.shard_info(g) for g in range(G)]
            assert [o[0] for o in offs] == [0] * G
            assert offs[0][1] == 0 and sum(o[2] for o in offs) == n
            for g in range(1, G):
                assert offs[g][1] == offs[g - 1][1] + offs[g - 1][2]
            sw = synth.ints_to_words(ks, S_W[name]) if n else np.zeros((0, S_W[name]), np.uint32)
            assert ctx.run(sw) == (closed(name, ks, es) if n else (0, 0)), (n, G)
        finally:
            ctx.close()


@pytest.mark.parametrize("G", [2, 4, 8])
def test_logical_shards_2p16_device_and_host_scalars(lib, G):
    """n = 2^16 BLS12-381 over G logical shards: host scalars (one staging thread per
    shard) and device scalars (each shard reads its slice in place) give the closed form;
    the same holds with the f3 table off (per-window bucket sets + window combine)."""
    import torch
    name = "bls12_381"
    c = CURVES[name]
    n = 1 << 16
    pts, es = gen_device_points(lib, name, n, 53)
    ks_w = synth.scalars_range(c.r, 0, n, 54)
    want = ec.to_output(ec.mul(sum(k * e for k, e in zip(synth.words_to_ints(ks_w), es)) % c.r, c.G, c))
    ctx = lib.Context(name, pts, n=n, devices=[0] * G)
    try:
        assert ctx.run(ks_w) == want
        ks_d = torch.from_numpy(ks_w.view(np.int32)).cuda()
        assert ctx.run(ks_d) == want
        ctx.set_option(lib.OPT_PRECOMPUTE, 0)
        assert ctx.run(ks_d) == want
    finally:
        ctx.close()


def test_context_on_current_device_and_device_restored(lib):
    """msm_context_create binds shard 0 to the caller's current device; every call leaves
    the caller's current device as it was.  With >= 2 GPUs, contexts created under
    cuda:1 live on device 1 (every context used to land on device 0)."""
    import torch
    name = "bn254"
    c = CURVES[name]
    n = 257
    Ps, es, _, _ = progression(name, n, 55)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 56))
    sw = synth.ints_to_words(ks, 8)
    ndev = lib.device_count()
    for dev in range(min(ndev, 2)):
        torch.cuda.set_device(dev)
        ctx = lib.Context(name, points_to_words(list(Ps), name), n=n)
        assert ctx.get_option(lib.OPT_DEVICE) == dev
        assert ctx.shard_info(0)[0] == dev
        assert torch.cuda.current_device() == dev
        assert ctx.run(sw) == closed(name, ks, es)
        assert torch.cuda.current_device() == dev
        ctx.close()
        assert torch.cuda.current_device() == dev
    torch.cuda.set_device(0)
    if ndev >= 2:
        ctx = lib.Context(name, points_to_words(list(Ps), name), n=n, ngpus=2)
        assert [ctx.shard_info(g)[0] for g in range(2)] == [0, 1]
        assert ctx.run(sw) == closed(name, ks, es)
        ctx.close()
    with pytest.raises(lib.MSMError) as e:
        lib.Context(name, points_to_words(list(Ps), name), n=n, devices=[ndev])
    assert e.value.code == -9


def test_device_inputs_ordered_after_default_stream(lib):
    """Scalars written by torch on its default stream right before msm_run (behind a long
    kernel) are what the MSM reads: the library orders itself after the legacy stream."""
    import torch
    name = "bls12_381"
    c = CURVES[name]
    n = 4096
    pts, es = gen_device_points(lib, name, n, 57)
    ks_a = synth.scalars_range(c.r, 0, n, 58)
    ks_b = synth.scalars_range(c.r, 0, n, 59)
    want_b = ec.to_output(ec.mul(sum(k * e for k, e in zip(synth.words_to_ints(ks_b), es)) % c.r, c.G, c))
    ctx = lib.Context(name, pts, n=n)
    buf = torch.from_numpy(ks_a.view(np.int32)).cuda()
    src = torch.from_numpy(ks_b.view(np.int32)).cuda()
    big = torch.randn(8192, 8192, device="cuda")
    for _ in range(3):
        torch.cuda.synchronize()
        big = big @ big / 8192.0      # keeps the default stream busy
        buf.copy_(src)                # the write the MSM must see
        assert ctx.run(buf) == want_b
        buf.copy_(torch.from_numpy(ks_a.view(np.int32)).cuda())
    ctx.close()


def test_headline_defaults_2p20(lib):
    """BLS12-381, n = 2^20, all defaults (automatic c and f3 table, staged sort chosen
    automatically, lockstep accumulation with ~thousands-entry slices): bit-exact."""
    name = "bls12_381"
    c = CURVES[name]
    n = 1 << 20
    pts, es = gen_device_points(lib, name, n, 60)
    ks_w = synth.scalars_range(c.r, 0, n, 61)
    ks = synth.words_to_ints(ks_w)
    want = ec.to_output(ec.mul(sum(k * e for k, e in zip(ks, es)) % c.r, c.G, c))
    ctx = lib.Context(name, pts, n=n)
    try:
        got = ctx.run(ks_w)
        st = ctx.stats()
        assert ctx.get_option(lib.OPT_SORT) == 3, "staged sort not auto-selected"
        assert ctx.get_option(lib.OPT_PRECOMPUTE) == 1
        assert st["entries"] >= (1 << 21)
        assert got == want
    finally:
        ctx.close()


@pytest.mark.slow
def test_bench_gpus2_self_launch():
    """`python bench.py --gpus 2` without torchrun: bench.py re-launches itself with two
    ranks (shared-device mode when the box has one GPU) and rank 0 prints one JSON line
    whose closed-form check passes."""
    for split in ("auto", "buckets"):  # auto = point shards in shared-device mode; buckets = f1
        cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--log2n", "16", "--steps", "2",
               "--warmup", "3", "--no-cpu-baseline", "--no-e2e", "--split", split]
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
        assert r.returncode == 0, r.stderr[-3000:]
        lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
        assert len(lines) == 1, r.stdout
        line = json.loads(lines[0])
        assert line["n_gpus"] == 2
        assert line["check"]["closed_form_match"] is True, split


@pytest.mark.parametrize("sort", [3, 4])
@pytest.mark.parametrize("kind,cbits,pre", [("equal", 13, 1), ("skewed", 16, 1), ("uniform", 8, 1),
                                            ("uniform", 16, 1), ("uniform", 12, 0)])
def test_cluster_sort_heavy_bins(lib, kind, cbits, pre, sort):
    """Two-pass cluster sort (sort4.cuh) at n = 2^18 where bins exceed one cluster round
    (S4_CL * S4_CAP = 196 608 entries): equal / skewed scalars put every entry in a few
    buckets, c = 8 makes bins of 8 buckets holding ~2^20 entries each; the histogram sweep
    and the rounds with running offsets must reproduce the closed form bit-exactly.  The
    same inputs through the staged sort (3) exercise its oversized sub-bins (k_s3_big)."""
    name = "bls12_381"
    c = CURVES[name]
    n = 1 << 18
    pts, es = gen_device_points(lib, name, n, 70)
    ks_w = (synth.scalars_range(c.r, 0, n, 71) if kind == "uniform"
            else synth.pattern_scalars(c.r, n, 72, kind))
    ks = synth.words_to_ints(ks_w)
    want = ec.to_output(ec.mul(sum(k * e for k, e in zip(ks, es)) % c.r, c.G, c))
    ctx = lib.Context(name, pts, n=n)
    try:
        ctx.set_option(lib.OPT_SORT, sort)
        ctx.set_option(lib.OPT_PRECOMPUTE, pre)
        ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
        assert ctx.get_option(lib.OPT_SORT) == sort
        assert ctx.run(ks_w) == want
    finally:
        ctx.close()


@pytest.mark.parametrize("pre", [1, 0])
def test_chunked_host_scalars(lib, pre):
    """Host scalars uploaded in K growing chunks, each sorted and accumulated INTO the
    bucket set (INIT accumulation): bit-exact against the closed form for
    K = 1..5 (auto = 1 below 2^22 points), with the f3 table on and off, BLS12-381
    n = 2^20; device scalars are never chunked."""
    name = "bls12_381"
    c = CURVES[name]
    n = 1 << 20
    pts, es = gen_device_points(lib, name, n, 80)
    ks_w = synth.scalars_range(c.r, 0, n, 81)
    ks = synth.words_to_ints(ks_w)
    ks_w[5] = 0                       # a zero scalar inside the first chunk
    ks[5] = 0
    want = ec.to_output(ec.mul(sum(k * e for k, e in zip(ks, es)) % c.r, c.G, c))
    ctx = lib.Context(name, pts, n=n)
    try:
        ctx.set_option(lib.OPT_PRECOMPUTE, pre)
        for K, used in ((0, 1), (1, 1), (2, 2), (3, 3), (4, 4), (5, 5)):  # auto: K = 3 from 2^22
            ctx.set_option(lib.OPT_H2D_CHUNKS, K)
            assert ctx.run(ks_w) == want, K
            assert ctx.get_option(lib.OPT_H2D_CHUNKS) == used
        import torch
        assert ctx.run(torch.from_numpy(ks_w.view(np.int32)).cuda()) == want
        assert ctx.get_option(lib.OPT_H2D_CHUNKS) == 1
    finally:
        ctx.close()
    # two logical shards on one device, each uploading its half in 3 chunks from its own
    # host thread and copy stream (f3 table on)
    ctx = lib.Context(name, pts, n=n, devices=[0, 0])
    try:
        ctx.set_option(lib.OPT_PRECOMPUTE, pre)
        ctx.set_option(lib.OPT_H2D_CHUNKS, 3)
        assert ctx.run(ks_w) == want
        assert ctx.get_option(lib.OPT_H2D_CHUNKS) == 3
    finally:
        ctx.close()


def test_small_n_autotune(lib):
    """Contexts of 2^10..2^17 points with automatic c measure the candidate window sizes at
    creation and keep the fastest (engine.cu autotune_c): the chosen c is one of the
    candidates, results stay bit-exact, and an explicit c still wins over the tuned one."""
    name = "bn254"
    c = CURVES[name]
    n = 1 << 12
    pts, es = gen_device_points(lib, name, n, 90)
    ks_w = synth.scalars_range(c.r, 0, n, 91)
    ks = synth.words_to_ints(ks_w)
    want = ec.to_output(ec.mul(sum(k * e for k, e in zip(ks, es)) % c.r, c.G, c))
    ctx = lib.Context(name, pts, n=n)
    try:
        tuned = ctx.get_option(lib.OPT_WINDOW_BITS)
        assert 4 <= tuned <= 16
        assert ctx.run(ks_w) == want
        ctx.set_option(lib.OPT_WINDOW_BITS, 9)
        assert ctx.get_option(lib.OPT_WINDOW_BITS) == 9
        assert ctx.run(ks_w) == want
        ctx.set_option(lib.OPT_WINDOW_BITS, 0)
        assert ctx.get_option(lib.OPT_WINDOW_BITS) == tuned
    finally:
        ctx.close()


def test_graph_replay_small_n(lib):
    """Small-n CUDA-graph replay (MSM_OPT_GRAPH): the graph is captured the second time the
    same device scalar buffer is seen; overwriting the buffer's CONTENTS between replays must
    change the result (kernels read memory at replay), a different buffer must not reuse the
    graph, stage times of a replayed run read -1 while the total stays valid, and
    MSM_OPT_GRAPH = 0 gives the same results through plain launches."""
    import torch
    name = "bn254"
    c = CURVES[name]
    n = 1 << 11
    pts, es = gen_device_points(lib, name, n, 95)
    ka = synth.scalars_range(c.r, 0, n, 96)
    kb = synth.scalars_range(c.r, 0, n, 97)

    def want(kw):
        ks = synth.words_to_ints(kw)
        return ec.to_output(ec.mul(sum(k * e for k, e in zip(ks, es)) % c.r, c.G, c))

    wa, wb = want(ka), want(kb)
    buf = torch.from_numpy(ka.view(np.int32)).cuda()
    other = torch.from_numpy(kb.view(np.int32)).cuda()
    ctx = lib.Context(name, pts, n=n)
    try:
        assert ctx.get_option(lib.OPT_GRAPH) == 1
        for _ in range(3):                       # launch, capture, replay
            assert ctx.run(buf) == wa
        st = ctx.stats()
        assert st["total_ms"] > 0 and st["accumulate_ms"] == -1.0
        buf.copy_(other)                         # same pointer, new contents
        assert ctx.run(buf) == wb
        assert ctx.run(torch.from_numpy(ka.view(np.int32)).cuda()) == wa   # other buffer
        ctx.set_option(lib.OPT_GRAPH, 0)
        assert ctx.run(buf) == wb
        assert ctx.stats()["accumulate_ms"] > 0
    finally:
        ctx.close()
