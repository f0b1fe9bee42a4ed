"""World-size-2 gloo tests of the multi-process host logic (no GPU): shard bounds cover
[0, n) exactly, per-rank scalar slices equal the slices of the full vector, the partial
gather returns rank-ordered partials, and — with the oracle standing in for the GPU
partial sums — the sum of per-shard MSMs equals the whole MSM (split invariance, the
identity the sharded path relies on)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_ji0x024_b200.dist import gather_partials, shard_bounds


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from oracle import ec, msm as omsm, points as opoints
        from oracle.curves import CURVES
        c = CURVES["bn254"]
        n = 37
        off, cnt = shard_bounds(n, world, rank)
        ks_full = synth.scalars_range(c.r, 0, n, 5)
        ks = synth.scalars_range(c.r, off, cnt, 5)
        assert np.array_equal(ks, ks_full[off:off + cnt])
        e0, d = synth.point_seeds(c.r, 9)
        Ps = opoints.progression_points(synth.progression_offset(c.r, e0, d, off), d, cnt, c)
        Q = omsm.msm_naive(synth.words_to_ints(ks), Ps, c)
        x, y = ec.to_output(Q)
        words = torch.tensor([(x >> (32 * i)) & 0xFFFFFFFF for i in range(8)] +
                             [(y >> (32 * i)) & 0xFFFFFFFF for i in range(8)], dtype=torch.int64).to(torch.int32)
        allp = gather_partials(words)
        if rank == 0:
            tot = None
            for r_ in range(world):
                w = allp[r_].to(torch.int64) & 0xFFFFFFFF
                px = sum(int(w[i]) << (32 * i) for i in range(8))
                py = sum(int(w[8 + i]) << (32 * i) for i in range(8))
                tot = ec.add(tot, None if (px, py) == (0, 0) else (px, py), c)
            Ps_all = opoints.progression_points(e0, d, n, c)
            full = omsm.msm_naive(synth.words_to_ints(ks_full), Ps_all, c)
            q.put(("ok", tot == full, [shard_bounds(n, world, r_) for r_ in range(world)]))
    except Exception as ex:  # pragma: no cover
        q.put(("err", repr(ex), None))
    finally:
        dist.destroy_process_group()


def test_shard_bounds_cover():
    for n in (0, 1, 5, 37, 1 << 20):
        for w in (1, 2, 3, 8):
            spans = [shard_bounds(n, w, r) for r in range(w)]
            assert spans[0][0] == 0
            assert sum(c for _, c in spans) == n
            assert all(spans[i][0] + spans[i][1] == spans[i + 1][0] for i in range(w - 1))


def test_two_rank_gather_and_split_invariance():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = q.get(timeout=240)
    for p in ps:
        p.join(timeout=60)
    assert res[0] == "ok", res
    assert res[1] is True
    assert res[2] == [(0, 18), (18, 19)]


def _worker_buckets(rank, world, port, q):
    """f1 bucket split: every rank holds ALL points and scalars and owns the
    buckets b = |d| with b mod world = rank; the oracle's part stands in for the GPU partial."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from oracle import ec, msm as omsm, points as opoints, stages
        from oracle.curves import CURVES
        c = CURVES["bn254"]
        n = 23
        ks = synth.words_to_ints(synth.scalars_range(c.r, 0, n, 12))
        e0, d = synth.point_seeds(c.r, 13)
        Ps = opoints.progression_points(e0, d, n, c)
        x, y = ec.to_output(stages.bucket_split_partial(ks, Ps, 5, c, world, rank, pre=False))
        words = torch.tensor([(x >> (32 * i)) & 0xFFFFFFFF for i in range(8)] +
                             [(y >> (32 * i)) & 0xFFFFFFFF for i in range(8)], dtype=torch.int64).to(torch.int32)
        allp = gather_partials(words)
        if rank == 0:
            tot = None
            for r_ in range(world):
                w = allp[r_].to(torch.int64) & 0xFFFFFFFF
                px = sum(int(w[i]) << (32 * i) for i in range(8))
                py = sum(int(w[8 + i]) << (32 * i) for i in range(8))
                tot = ec.add(tot, None if (px, py) == (0, 0) else (px, py), c)
            q.put(("ok", tot == omsm.msm_naive(ks, Ps, c), None))
    except Exception as ex:  # pragma: no cover
        q.put(("err", repr(ex), None))
    finally:
        dist.destroy_process_group()


def test_two_rank_bucket_split():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker_buckets, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = q.get(timeout=240)
    for p in ps:
        p.join(timeout=60)
    assert res[0] == "ok", res
    assert res[1] is True
