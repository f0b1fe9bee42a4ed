"""End-to-end parity of the CUDA MSM (through the C-ABI) with the oracle: bit-exact
affine results for every curve over ragged sizes, several window sizes, edge cases and
adversarial inputs; stage-level parity of bucket sums and window sums; error paths."""
import numpy as np
import pytest

import synth
from oracle import ec, msm as omsm, stages
from oracle.curves import CURVES
from tests.helpers import L32, S_W, points_to_words, progression

pytestmark = pytest.mark.gpu
NAMES = ["bn254", "bls12_377", "bls12_381", "mnt4_753"]


@pytest.fixture(scope="module")
def lib():
    from paper_conf_asplos_ji0x024_b200 import msm as m
    assert m.device_count() >= 1, "no CUDA device"
    return m


def closed(name, ks, es):
    return ec.to_output(omsm.msm_closed_form(ks, es, CURVES[name]))


def run(lib, name, Ps, ks, c=None, ngpus=1, pre=None):
    ctx = lib.Context(name, points_to_words(Ps, name), ngpus=ngpus, n=len(Ps))
    try:
        if pre is not None:
            ctx.set_option(lib.OPT_PRECOMPUTE, pre)
        if c:
            ctx.set_option(lib.OPT_WINDOW_BITS, c)
        return ctx.run(synth.ints_to_words(ks, S_W[name]) if ks else np.zeros((0, S_W[name]), np.uint32))
    finally:
        ctx.close()


@pytest.mark.parametrize("name", NAMES)
@pytest.mark.parametrize("n", [1, 2, 3, 7, 31, 33, 255, 1025])
def test_msm_ragged_sizes(lib, name, n):
    if name == "mnt4_753" and n > 255:
        n = 129
    c = CURVES[name]
    Ps, es, _, _ = progression(name, n, 21)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 1000 + n))
    assert run(lib, name, list(Ps), ks) == closed(name, ks, es)


@pytest.mark.parametrize("name", ["bn254", "bls12_381", "mnt4_753"])
@pytest.mark.parametrize("cbits", [2, 3, 4, 7, 11, 16])
def test_msm_window_sizes(lib, name, cbits):
    c = CURVES[name]
    n = 96 if name != "mnt4_753" else 40
    if name == "mnt4_753" and cbits < 4:
        pytest.skip("too many windows for a quick test")
    Ps, es, _, _ = progression(name, n, 22)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 7 * cbits))
    assert run(lib, name, list(Ps), ks, c=cbits) == closed(name, ks, es)


def test_msm_n0(lib):
    for name in NAMES:
        assert run(lib, name, [], []) == (0, 0)


@pytest.mark.parametrize("name", NAMES)
@pytest.mark.parametrize("kind", ["zeros", "ones", "max", "equal", "skewed", "extremes"])
def test_msm_patterns(lib, name, kind):
    c = CURVES[name]
    n = 200 if name != "mnt4_753" else 60
    Ps, es, _, _ = progression(name, n, 23)
    ks = synth.words_to_ints(synth.pattern_scalars(c.r, n, 5, kind))
    assert run(lib, name, list(Ps), ks, c=6) == closed(name, ks, es)


@pytest.mark.parametrize("name", NAMES)
def test_msm_adversarial_points(lib, name):
    """Duplicate points in one bucket (forces doubling in PACC), k and r-k on the same
    point (cancellation to O inside a bucket), consecutive multiples iG, O points."""
    c = CURVES[name]
    G = c.G
    Ps = [G] * 6 + [ec.mul(i + 1, G, c) for i in range(10)] + [None, None]
    ks = [5, 5, 5, c.r - 5, 3, c.r - 3] + [i + 1 for i in range(10)] + [7, c.r - 1]
    es = [1] * 6 + [i + 1 for i in range(10)]
    want = ec.to_output(ec.mul(sum(k * e for k, e in zip(ks, es)) % c.r, G, c))
    for cbits in (3, 4, 8):
        assert run(lib, name, Ps, ks, c=cbits) == want, cbits
    # all points equal: (sum k) * P
    P = ec.mul(12345, G, c)
    ks2 = synth.words_to_ints(synth.scalars(c.r, 64, 9))
    assert run(lib, name, [P] * 64, ks2, c=5) == ec.to_output(ec.mul(sum(ks2) % c.r, P, c))


@pytest.mark.parametrize("name", ["bn254", "bls12_381", "mnt4_753"])
def test_stage_parity_buckets_and_windows(lib, name):
    """Every bucket sum B_{j,b} and window sum W_j equals the oracle's staged model."""
    c = CURVES[name]
    n = 150 if name != "mnt4_753" else 50
    cbits = 5
    Ps, es, _, _ = progression(name, n, 24)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 77))
    ctx = lib.Context(name, points_to_words(list(Ps), name), n=n)
    ctx.set_option(lib.OPT_PRECOMPUTE, 0)
    ctx.set_option(1, cbits)
    assert ctx.get_option(lib.OPT_NSETS) == ctx.get_option(lib.OPT_NWIN)
    Ws, Bs = ctx.windows(synth.ints_to_words(ks, S_W[name]), with_buckets=True)
    ctx.close()
    Bo = stages.bucket_sums(ks, list(Ps), cbits, c)
    Wo = stages.window_sums(Bo, c)
    assert len(Ws) == len(Wo)
    for j in range(len(Wo)):
        assert Ws[j] == ec.to_output(Wo[j]), j
        for b in range(1, len(Bo[j])):
            assert Bs[j][b] == ec.to_output(Bo[j][b]), (j, b)


@pytest.mark.parametrize("name", NAMES)
def test_split_invariance_and_partials(lib, name):
    """MSM[0,n) = MSM[0,m) + MSM[m,n): two contexts' XYZZ partials through msm_finalize."""
    c = CURVES[name]
    n, m = 120, 47
    Ps, es, _, _ = progression(name, n, 25)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 31))
    pw = lib.partial_words(name)
    parts = np.zeros(2 * pw, dtype=np.uint32)
    for g, (a, b) in enumerate([(0, m), (m, n)]):
        ctx = lib.Context(name, points_to_words(list(Ps[a:b]), name), n=b - a)
        ctx.run_partial(synth.ints_to_words(ks[a:b], S_W[name]), parts[g * pw:(g + 1) * pw])
        ctx.close()
    assert lib.finalize(name, parts, 2) == closed(name, ks, es)
    assert lib.finalize(name, parts, 0) == (0, 0)


def test_errors(lib):
    name = "bls12_381"
    c = CURVES[name]
    Ps, es, _, _ = progression(name, 8, 26)
    Pw = points_to_words(list(Ps), name)
    ctx = lib.Context(name, Pw, n=8)
    ks = synth.words_to_ints(synth.scalars(c.r, 8, 1))
    bad = list(ks)
    bad[3] = c.r
    with pytest.raises(lib.MSMError) as e:
        ctx.run(synth.ints_to_words(bad, 8))
    assert e.value.code == -7
    assert ctx.run(synth.ints_to_words(ks, 8)) == closed(name, ks, es)  # still usable
    ctx.close()
    Pw2 = Pw.copy()
    Pw2[2, 0] ^= 1  # off the curve
    with pytest.raises(lib.MSMError) as e:
        lib.Context(name, Pw2, n=8)
    assert e.value.code == -6
    with pytest.raises(lib.MSMError) as e:
        lib.Context(name, Pw, ngpus=lib.device_count() + 1, n=8)
    assert e.value.code == -9


def test_device_resident_inputs(lib):
    """Points and scalars given as CUDA tensors (torch used only for device memory)."""
    import torch
    name = "bls12_381"
    c = CURVES[name]
    n = 300
    Ps, es, _, _ = progression(name, n, 27)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 2))
    Pt = torch.from_numpy(points_to_words(list(Ps), name).view(np.int32)).cuda()
    St = torch.from_numpy(synth.ints_to_words(ks, 8).view(np.int32)).cuda()
    ctx = lib.Context(name, Pt, n=n)
    assert ctx.run(St) == closed(name, ks, es)
    st = ctx.stats()
    assert st["h2d_ms"] >= 0 and st["accumulate_ms"] > 0
    ctx.close()


@pytest.mark.parametrize("name", ["bn254", "bls12_381"])
@pytest.mark.parametrize("sort", [1, 2, 3, 4])
@pytest.mark.parametrize("cbits", [4, 9, 13, 16])
def test_sort_variants(lib, name, sort, cbits):
    """a3 variants -- direct atomics (ablation), two-level binned, three-level staged,
    two-pass cluster -- all give the oracle's result and the oracle's bucket sums, for bin
    shifts 0..> 0."""
    c = CURVES[name]
    n = 700
    Ps, es, _, _ = progression(name, n, 28)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 40 + cbits))
    ctx = lib.Context(name, points_to_words(list(Ps), name), n=n)
    ctx.set_option(lib.OPT_PRECOMPUTE, 0)
    ctx.set_option(lib.OPT_SORT, sort)
    ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
    assert ctx.get_option(lib.OPT_SORT) == sort
    sw = synth.ints_to_words(ks, S_W[name])
    assert ctx.run(sw) == closed(name, ks, es)
    if cbits <= 9:
        Ws, Bs = ctx.windows(sw, with_buckets=True)
        Bo = stages.bucket_sums(ks, list(Ps), cbits, c)
        for j in range(len(Bo)):
            for b in range(1, len(Bo[j])):
                assert Bs[j][b] == ec.to_output(Bo[j][b]), (j, b)
    ctx.close()


def test_large_c_binned_sort(lib):
    """c = 20..22 (the bench's windows): shift > 0 bins, many empty buckets at small n."""
    name = "bls12_381"
    c = CURVES[name]
    n = 3000
    Ps, es, _, _ = progression(name, n, 29)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 41))
    ctx = lib.Context(name, points_to_words(list(Ps), name), n=n)
    for sort in (2, 3, 4):
        ctx.set_option(lib.OPT_SORT, sort)
        for pre in (0, 1):
            ctx.set_option(lib.OPT_PRECOMPUTE, pre)
            for cbits in (20, 22, 24):
                ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
                assert ctx.run(synth.ints_to_words(ks, 8)) == closed(name, ks, es), (sort, pre, cbits)
    ctx.close()


@pytest.mark.parametrize("sort", [3, 4])
@pytest.mark.parametrize("kind", ["ones", "skewed", "uniform"])
def test_staged_sort_oversized_subbins(lib, kind, sort):
    """Staged sorts on skewed scalars: three-level with > S3_CAP entries in one sub-bin (the
    global-scatter fallback of k_s3_part3), two-pass cluster with bins of a few buckets;
    and on uniform scalars at several c."""
    name = "bn254"
    c = CURVES[name]
    n = 20000
    Ps, es, _, _ = progression(name, n, 34)
    ks = (synth.words_to_ints(synth.scalars(c.r, n, 62)) if kind == "uniform"
          else synth.words_to_ints(synth.pattern_scalars(c.r, n, 7, kind)))
    want = closed(name, ks, es)
    ctx = lib.Context(name, points_to_words(list(Ps), name), n=n)
    ctx.set_option(lib.OPT_SORT, sort)
    sw = synth.ints_to_words(ks, 8)
    for pre in (0, 1):
        ctx.set_option(lib.OPT_PRECOMPUTE, pre)
        for cbits in (5, 11, 16):
            ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
            assert ctx.get_option(lib.OPT_SORT) == sort
            assert ctx.run(sw) == want, (pre, cbits)
    ctx.close()


@pytest.mark.parametrize("name", NAMES)
def test_precompute_modes(lib, name):
    """f3 table on / off / auto: same result (closed form) at several c,
    ragged n, with O points and duplicates; the option reports the mode in use."""
    c = CURVES[name]
    n = 257 if name != "mnt4_753" else 65
    Ps, es, _, _ = progression(name, n, 30)
    Ps = list(Ps)
    Ps[5] = None          # O in the table stays O
    Ps[9] = Ps[8]         # duplicate point: doubling inside a shared bucket
    ks = synth.words_to_ints(synth.scalars(c.r, n, 51))
    ks[8], ks[9] = ks[9], ks[9]
    e = [0 if P is None else x for P, x in zip(Ps, es)]
    e[9] = es[8]
    want = closed(name, ks, e)
    ctx = lib.Context(name, points_to_words(Ps, name), n=n)
    sw = synth.ints_to_words(ks, S_W[name])
    for pre in (1, 0, 2):
        ctx.set_option(lib.OPT_PRECOMPUTE, pre)
        for cbits in ((3, 8, 13) if name != "mnt4_753" else (6, 11)):
            ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
            assert ctx.run(sw) == want, (pre, cbits)
            if pre != 2:
                assert ctx.get_option(lib.OPT_PRECOMPUTE) == pre
                assert ctx.get_option(lib.OPT_NSETS) == (1 if pre else ctx.get_option(lib.OPT_NWIN))
        ctx.set_option(lib.OPT_WINDOW_BITS, 0)
        assert ctx.run(sw) == want, (pre, "auto c")
    assert ctx.stats()["precompute"] in (0, 1)
    ctx.close()


@pytest.mark.parametrize("name", ["bn254", "bls12_377", "mnt4_753"])
def test_stage_parity_precomputed(lib, name):
    """With the f3 table: every bucket sum of the single shared set equals the oracle's
    B^pre_b = sum over (i, j) of sgn(d_ij) 2^(jc) P_i, and its reduce is the MSM."""
    c = CURVES[name]
    n = 90 if name != "mnt4_753" else 30
    cbits = 6 if name != "mnt4_753" else 9
    Ps, es, _, _ = progression(name, n, 31)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 78))
    ctx = lib.Context(name, points_to_words(list(Ps), name), n=n)
    ctx.set_option(lib.OPT_PRECOMPUTE, 1)
    ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
    assert ctx.get_option(lib.OPT_NSETS) == 1
    Ws, Bs = ctx.windows(synth.ints_to_words(ks, S_W[name]), with_buckets=True)
    ctx.close()
    Bo = stages.bucket_sums_precomputed(ks, list(Ps), cbits, c)
    for b in range(1, len(Bo)):
        assert Bs[0][b] == ec.to_output(Bo[b]), b
    assert Ws == [closed(name, ks, es)]


@pytest.mark.parametrize("name", ["bn254", "bls12_381"])
@pytest.mark.parametrize("kind", ["ones", "equal", "skewed"])
def test_fixup_long_runs(lib, name, kind):
    """Heavy buckets spanning many accumulation slices (skewed scalars, many threads):
    k_fixup hands runs of > 8 carries to k_fixup_long's block tree."""
    c = CURVES[name]
    n = 3000
    Ps, es, _, _ = progression(name, n, 32)
    ks = synth.words_to_ints(synth.pattern_scalars(c.r, n, 6, kind))
    want = closed(name, ks, es)
    ctx = lib.Context(name, points_to_words(list(Ps), name), n=n)
    sw = synth.ints_to_words(ks, S_W[name])
    for pre in (0, 1):
        ctx.set_option(lib.OPT_PRECOMPUTE, pre)
        ctx.set_option(lib.OPT_WINDOW_BITS, 8)
        for threads in (1, 37, 4096, 20000):
            ctx.set_option(lib.OPT_ACC_THREADS, threads)
            assert ctx.run(sw) == want, (pre, threads)
    ctx.close()


@pytest.mark.parametrize("cbits", [15, 17])
def test_degenerate_top_window(lib, cbits):
    """c dividing 255: the top window holds only the carry digit (bucket 1 gets ~n/2
    entries) -- correct and not serialised in k_fixup."""
    name = "bls12_381"
    c = CURVES[name]
    n = 4000
    Ps, es, _, _ = progression(name, n, 33)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 61))
    ctx = lib.Context(name, points_to_words(list(Ps), name), n=n)
    ctx.set_option(lib.OPT_PRECOMPUTE, 0)
    ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
    assert ctx.run(synth.ints_to_words(ks, 8)) == closed(name, ks, es)
    ctx.close()


@pytest.mark.parametrize("name", ["bn254", "bls12_381", "mnt4_753"])
@pytest.mark.parametrize("pre", [0, 1])
def test_bucket_split_parity(lib, name, pre):
    """f1 bucket split: G contexts over ALL points, context g summing only
    the buckets |d| = G*q + g.  Each part's partial (affine through msm_finalize) equals the
    oracle's part (stages.bucket_split_partial, computed from the definition), and the G
    partials finalize to the closed form.  Ragged n, G not dividing 2^(c-1), O points and
    duplicates (doubling inside a part)."""
    c = CURVES[name]
    n = 45 if name == "mnt4_753" else 131
    Ps, es, _, _ = progression(name, n, 41)
    Ps = list(Ps)
    Ps[2] = None
    Ps[7] = Ps[6]
    ks = synth.words_to_ints(synth.scalars(c.r, n, 43))
    ks[6] = ks[7]
    e = [0 if P is None else x for P, x in zip(Ps, es)]
    e[7] = es[6]
    sw = synth.ints_to_words(ks, S_W[name])
    pw = lib.partial_words(name)
    for cbits, G in ((5, 3), (7, 2), (6, 5)):
        parts = np.zeros(G * pw, dtype=np.uint32)
        for g in range(G):
            ctx = lib.Context(name, points_to_words(Ps, name), n=n)
            ctx.set_option(lib.OPT_PRECOMPUTE, pre)
            ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
            ctx.set_option(lib.OPT_SPLIT_PARTS, G)
            ctx.set_option(lib.OPT_SPLIT_INDEX, g)
            assert ctx.get_option(lib.OPT_SPLIT_PARTS) == G and ctx.get_option(lib.OPT_SPLIT_INDEX) == g
            ctx.run_partial(sw, parts[g * pw:(g + 1) * pw])
            ctx.close()
            want_g = ec.to_output(stages.bucket_split_partial(ks, Ps, cbits, c, G, g, bool(pre)))
            assert lib.finalize(name, parts[g * pw:(g + 1) * pw], 1) == want_g, (cbits, G, g)
        assert lib.finalize(name, parts, G) == closed(name, ks, e), (cbits, G)


def test_bucket_split_large_balanced(lib):
    """f1 at a size that uses the staged sort and many segments: BLS12-381, n = 2^16, auto c
    with the f3 table, G = 4 parts finalize to the closed form, and the interleaved
    assignment keeps every part's entry count within 3 % of the mean."""
    name = "bls12_381"
    c = CURVES[name]
    n = 1 << 16
    e0, d = synth.point_seeds(c.r, 77)
    import torch
    pts = torch.empty((n, 2 * L32[name]), dtype=torch.int32, device="cuda")
    lib.gen_points(name, e0, d, n, pts)
    ks = synth.scalars_range(c.r, 0, n, 78)
    es_sum = sum(k * ((e0 + i * d) % c.r) for i, k in enumerate(synth.words_to_ints(ks))) % c.r
    want = ec.to_output(ec.mul(es_sum, c.G, c))
    G = 4
    pw = lib.partial_words(name)
    parts = np.zeros(G * pw, dtype=np.uint32)
    entries = []
    for g in range(G):
        ctx = lib.Context(name, pts, n=n)
        ctx.set_option(lib.OPT_WINDOW_BITS, 14)  # the cost model's c (creation autotunes small n)
        ctx.set_option(lib.OPT_SPLIT_PARTS, G)
        ctx.set_option(lib.OPT_SPLIT_INDEX, g)
        ctx.run_partial(ks, parts[g * pw:(g + 1) * pw])
        entries.append(ctx.stats()["entries"])
        ctx.close()
    assert lib.finalize(name, parts, G) == want
    mean = sum(entries) / G
    # 3 %: at the planner's c = 14 the 3-bit top window's digits 1..8 fall unevenly on 4 parts
    assert max(abs(x - mean) for x in entries) < 0.03 * mean, entries


@pytest.mark.parametrize("name", ["bn254", "bls12_381", "mnt4_753"])
def test_pipelined_submit_wait(lib, name):
    """msm_submit / msm_wait: interleaved submissions (the next MSM's H2D overlaps the
    current one) give each MSM's own closed-form result; a scalar >= r fails only its own
    ticket; over-submission and out-of-order waits are rejected; the context stays usable
    and agrees with msm_run."""
    c = CURVES[name]
    n = 700 if name != "mnt4_753" else 90
    Ps, es, _, _ = progression(name, n, 61)
    ctx = lib.Context(name, points_to_words(Ps, name), n=n)
    sets = [synth.words_to_ints(synth.scalars(c.r, n, 70 + t)) for t in range(5)]
    bad = list(sets[3])
    bad[n // 2] = c.r  # k >= r
    words = [synth.ints_to_words(k, S_W[name]) for k in sets]
    words[3] = synth.ints_to_words(bad, S_W[name])
    t0 = ctx.submit(words[0])
    t1 = ctx.submit(words[1])
    with pytest.raises(lib.MSMError):
        ctx.submit(words[2])           # MSM_MAX_INFLIGHT = 2 outstanding
    with pytest.raises(lib.MSMError):
        ctx.wait(t1)                   # not the oldest outstanding ticket
    assert ctx.wait(t0) == closed(name, sets[0], es)
    t2 = ctx.submit(words[2])
    assert ctx.wait(t1) == closed(name, sets[1], es)
    t3 = ctx.submit(words[3])
    assert ctx.wait(t2) == closed(name, sets[2], es)
    t4 = ctx.submit(words[4])
    with pytest.raises(lib.MSMError) as ei:
        ctx.wait(t3)
    assert ei.value.code == -7         # MSM_ERR_SCALAR, this ticket only
    assert ctx.wait(t4) == closed(name, sets[4], es)
    assert ctx.run(words[1]) == closed(name, sets[1], es)
    t5 = ctx.submit(words[0])
    assert ctx.wait(t5) == closed(name, sets[0], es)
    ctx.close()


@pytest.mark.parametrize("name", ["bn254", "bls12_377", "bls12_381"])
@pytest.mark.parametrize("pre", [0, 1])
def test_batch_affine_front_end(lib, name, pre):
    """a4 batch-affine front end (MSM_OPT_ACC_MODE = 1; baff.cuh): every group of up to 4
    entries of a bucket is folded by pairwise affine additions sharing one inversion per
    batch.  Exercised on buckets of every size mod 4, pairs that double (equal points, equal
    digits), pairs that cancel (k and r - k on one point), O points inside groups, and many
    batches per thread (few threads forced through MSM_OPT_ACC_THREADS does not apply to the
    front end, so small c packs long buckets).  Bit-exact vs the closed form, and equal to
    the PACC-only path (mode 0)."""
    c = CURVES[name]
    G = c.G
    base = [ec.mul(i + 2, G, c) for i in range(40)]
    Ps, es, ks = [], [], []
    rng = np.random.default_rng(7)
    for i in range(600):
        kind = i % 6
        j = int(rng.integers(0, 40))
        if kind == 0:      # duplicate of the previous point with the same scalar -> doubling pairs
            P, e, k = (Ps[-1], es[-1], ks[-1]) if Ps else (base[j], j + 2, 5)
        elif kind == 1:    # the previous point with r - k -> cancelling pairs
            P, e, k = (Ps[-1], es[-1], (c.r - ks[-1]) % c.r) if Ps else (base[j], j + 2, 7)
        elif kind == 2:    # O
            P, e, k = None, 0, int(rng.integers(1, 1 << 20))
        else:
            P, e, k = base[j], j + 2, int(rng.integers(1, 64))
        Ps.append(P)
        es.append(e)
        ks.append(k)
    want = ec.to_output(ec.mul(sum(k * e for k, e in zip(ks, es)) % c.r, G, c))
    ctx = lib.Context(name, points_to_words(Ps, name), n=len(Ps))
    sw = synth.ints_to_words(ks, S_W[name])
    try:
        try:
            ctx.set_option(lib.OPT_ACC_MODE, 1)
        except lib.MSMError as e:
            assert e.code == -8
            pytest.skip("batch-affine front end not built (tools/build.py -D MSM_BAFF=1)")
        ctx.set_option(lib.OPT_PRECOMPUTE, pre)
        for cbits in (3, 5, 7):
            ctx.set_option(lib.OPT_WINDOW_BITS, cbits)
            ctx.set_option(lib.OPT_ACC_MODE, 1)
            assert ctx.get_option(lib.OPT_ACC_MODE) == 1
            got1 = ctx.run(sw)
            st = ctx.stats()
            assert st["baff"] == 1 and st["entries_acc"] < st["entries"]
            ctx.set_option(lib.OPT_ACC_MODE, 0)
            assert ctx.get_option(lib.OPT_ACC_MODE) == 0
            got0 = ctx.run(sw)
            assert got1 == want, (cbits, "front end")
            assert got0 == want, (cbits, "PACC only")
    finally:
        ctx.close()
