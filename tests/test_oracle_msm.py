"""Pins for oracle/msm.py and oracle/stages.py: three independent MSM routes agree
(naive double-and-add, plain unsigned Pippenger, closed form), the staged signed-digit
decomposition the GPU follows equals them, and the signed-digit rule reconstructs k."""
import json
import os
import random

import pytest

from oracle import ec, msm, points, stages
from oracle.curves import CURVES
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")
ALL = list(CURVES.values())


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_appendix_d_vectors(c):
    g = json.load(open(os.path.join(GOLD, "known_points.json")))["msm_14G"][c.name]
    G = c.G
    Ps = [G, ec.double(G, c), ec.add(G, ec.double(G, c), c)]
    ks = [1, 2, 3]
    want = (int(g[0], 16), int(g[1], 16))
    assert msm.msm_naive(ks, Ps, c) == want
    assert msm.msm_pippenger(ks, Ps, c, s=4) == want
    assert stages.msm_staged(ks, Ps, 5, c) == want
    assert ec.mul(14, G, c) == want
    # (r-1)*G + 2*G == G
    assert msm.msm_naive([c.r - 1, 2], [G, G], c) == G
    assert stages.msm_staged([c.r - 1, 2], [G, G], 7, c) == G


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_three_routes_agree(c):
    n = 12 if c.name == "mnt4_753" else 24
    e0, d = synth.point_seeds(c.r, 4)
    Ps = points.progression_points(e0, d, n, c)
    es = points.progression_scalars(e0, d, n, c)
    assert all(ec.mul(e, c.G, c) == P for e, P in zip(es[:3], Ps[:3]))
    ks = synth.words_to_ints(synth.scalars(c.r, n, 99))
    ks[0] = 0
    ks[1] = c.r - 1
    ks[2] = 1
    want = msm.msm_closed_form(ks, es, c)
    assert msm.msm_naive(ks, Ps, c) == want
    assert msm.msm_pippenger(ks, Ps, c, s=5) == want
    for cc in (3, 4, 7, 13):
        assert stages.msm_staged(ks, Ps, cc, c) == want
    iks = sum(i * k for i, k in enumerate(ks))
    assert msm.closed_form_arith(sum(ks), iks, e0, d, c) == want


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_signed_digits(c):
    lam = c.lam
    ex = [0, 1, 2, c.r - 1, c.r - 2, 1 << (lam - 1), (1 << lam) - 1, (1 << (lam - 1)) - 1]
    rng = random.Random(5)
    ex += [rng.randrange(c.r) for _ in range(10)]
    for cc in range(2, 27):
        half = 1 << (cc - 1)
        for k in ex:
            ds = stages.signed_digits(k, lam, cc)
            assert len(ds) == lam // cc + 1
            assert sum(d << (j * cc) for j, d in enumerate(ds)) == k
            assert all(-half < d <= half for d in ds[:-1])
            assert 0 <= ds[-1] <= half


def test_staged_edge_cases():
    c = CURVES["bn254"]
    e0, d = synth.point_seeds(c.r, 8)
    Ps = points.progression_points(e0, d, 6, c)
    assert stages.msm_staged([], [], 4, c) is None
    assert stages.msm_staged([0] * 6, Ps, 4, c) is None
    # k and r-k on the same point cancel
    assert stages.msm_staged([5, c.r - 5], [Ps[0], Ps[0]], 4, c) is None
    # duplicate points in one bucket force doubling inside the bucket
    assert stages.msm_staged([3, 3, 3], [Ps[1]] * 3, 4, c) == ec.mul(9, Ps[1], c)
    # consecutive multiples i*G
    G = c.G
    Pm = [ec.mul(i + 1, G, c) for i in range(8)]
    ks = [i + 1 for i in range(8)]
    assert stages.msm_staged(ks, Pm, 3, c) == ec.mul(sum((i + 1) ** 2 for i in range(8)), G, c)


def test_synth_scalars_in_range():
    for c in ALL:
        ks = synth.words_to_ints(synth.scalars(c.r, 500, 1))
        assert all(0 <= k < c.r for k in ks)
        assert max(ks).bit_length() >= c.lam - 3


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_precomputed_route(c):
    """f3: the table rows are 2^(jc) P (checked with the library-style
    double-and-add ec.mul), the shared bucket set is sum_j 2^(jc) B_{j,b} of the per-window
    model, and its single bucket-reduce is the MSM (closed form)."""
    n = 6 if c.name == "mnt4_753" else 14
    e0, d = synth.point_seeds(c.r, 8)
    Ps = points.progression_points(e0, d, n, c)
    es = points.progression_scalars(e0, d, n, c)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 123))
    ks[0], ks[1] = c.r - 1, 0
    want = msm.msm_closed_form(ks, es, c)
    big = c.name == "mnt4_753"
    for cc in ((5, 9) if not big else (16,)):
        T = stages.precomputed_table(Ps[:2], cc, c)
        for j in (range(len(T)) if not big else (1, 2, len(T) - 1)):
            assert T[j][1] == ec.mul(pow(2, j * cc), Ps[1], c)
        Bp = stages.bucket_sums_precomputed(ks, Ps, cc, c)
        Bw = stages.bucket_sums(ks, Ps, cc, c)
        for b in (range(1, len(Bp)) if not big else ()):
            acc = None
            for j in range(len(Bw)):
                acc = ec.add(acc, ec.mul(pow(2, j * cc), Bw[j][b], c) if Bw[j][b] else None, c)
            assert Bp[b] == acc, b
        assert stages.msm_precomputed(ks, Ps, cc, c) == want


@pytest.mark.parametrize("c", [CURVES["bn254"], CURVES["bls12_381"]], ids=lambda c: c.name)
def test_bucket_split_parts_sum_to_msm(c):
    """f1 bucket split: the G parts' partials add up to the closed form for
    several G (incl. G not dividing 2^(c-1)) with and without the f3 table, and one part
    (G = 1) is the whole MSM.  A wrong weight, a dropped residue class or a part counted
    twice breaks the sum."""
    n = 20
    e0, d = synth.point_seeds(c.r, 6)
    Ps = points.progression_points(e0, d, n, c)
    es = points.progression_scalars(e0, d, n, c)
    ks = synth.words_to_ints(synth.scalars(c.r, n, 17))
    ks[3] = c.r - 1
    ks[4] = 1
    want = msm.msm_closed_form(ks, es, c)
    for pre in (False, True):
        for cc, G in ((5, 2), (5, 3), (6, 5), (4, 8)):
            parts = [stages.bucket_split_partial(ks, Ps, cc, c, G, g, pre) for g in range(G)]
            tot = None
            for P in parts:
                tot = ec.add(tot, P, c)
            assert tot == want, (pre, cc, G)
        assert stages.bucket_split_partial(ks, Ps, 5, c, 1, 0, pre) == want
    # a part is not the whole: with G = 2 both halves are generically non-trivial and differ
    h0 = stages.bucket_split_partial(ks, Ps, 5, c, 2, 0)
    h1 = stages.bucket_split_partial(ks, Ps, 5, c, 2, 1)
    assert h0 != h1 and h0 is not None and h1 is not None
