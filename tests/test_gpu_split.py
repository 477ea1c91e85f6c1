"""GPU parity of the launch split (-m gpu): a call with more points than one probe sub-launch
holds (< 2^31 points; spade_set_option "max_launch_points" lowers it for tests) runs several
sub-launches, each with its own deferral regions, output chunks and compaction, and spreads the
per-record counters of multi-owner / K-aggregated records over their owner sets after every
sub-launch (so a uint32 counter never sees 2^32 points).  Every op and every probe path must give
the oracle's result bit for bit whatever the split (aggregation exactness
P:214, capacity / n_max P:258).
"""
import numpy as np
import pytest

import gen
import oracle
from gen import configs
from tests.helpers import sorted_pairs

pytestmark = pytest.mark.gpu

DEFAULTS = {"defer": 0, "count_global": 0, "pipe": -1, "multi_agg": 1, "k_agg": -1, "max_launch_points": (1 << 31) - 64,
            "defer_budget_mb": 4096}


@pytest.fixture(scope="module")
def spade():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icde_doraiswamyf22_b200 as sp
    sp.load()
    yield sp
    for k, v in DEFAULTS.items():
        sp.set_option(k, v)


def _set(sp, opts):
    for k, v in DEFAULTS.items():
        sp.set_option(k, opts.get(k, v))


SPLITS = [{"max_launch_points": 256}, {"max_launch_points": 4099}, {"max_launch_points": 65536}]
PATHS = [{}, {"defer": 1}, {"pipe": 1}, {"count_global": 1}, {"k_agg": 1}, {"k_agg": 1, "defer": 1},
         {"multi_agg": 0, "k_agg": 1, "pipe": 1}, {"k_agg": 1, "count_global": 1, "defer": 1}]


def _ids(o):
    return ",".join(f"{k}={v}" for k, v in o.items()) or "default"


def _c1_case():
    w = configs.c1()
    xy = np.concatenate([gen.points_host(w.points, w.point_seed, 0, 60_000), configs.c1_edge_points(w.polys)])
    return w.polys, xy


def _overlap_case():
    w = configs.ov()
    return w.polys, gen.points_host(w.points, w.point_seed, 0, 40_000)


CASES = {"c1": _c1_case, "ov": _overlap_case}


@pytest.mark.parametrize("split", SPLITS, ids=_ids)
@pytest.mark.parametrize("path", PATHS, ids=_ids)
@pytest.mark.parametrize("case", list(CASES))
def test_count_split_matches_oracle(spade, case, path, split):
    import torch
    polys, xy = CASES[case]()
    _set(spade, {**path, **split})
    try:
        cv = spade.Canvas(polys, max_dim=1024 if case == "c1" else 4096)
        counts = spade.join_count(cv, torch.as_tensor(xy).cuda()).cpu().numpy()
    finally:
        _set(spade, {})
    np.testing.assert_array_equal(counts, oracle.join_count(xy, polys))


@pytest.mark.parametrize("split", SPLITS, ids=_ids)
@pytest.mark.parametrize("path", [{}, {"defer": 1}], ids=_ids)
@pytest.mark.parametrize("case", list(CASES))
def test_select_pairs_split_match_oracle(spade, case, path, split):
    """Each sub-launch hands out its own warp output chunks; the holes of every sub-launch are
    compacted before the next starts, so the output stays dense across the split."""
    import torch
    polys, xy = CASES[case]()
    _set(spade, {**path, **split})
    try:
        cv = spade.Canvas(polys, max_dim=1024 if case == "c1" else 4096)
        xy_d = torch.as_tensor(xy).cuda()
        cap = len(xy) if case == "c1" else None
        if case == "ov":
            cap = int(spade.join_count(cv, xy_d).sum())
        pt, pl = spade.join_pairs(cv, xy_d, point_id_base=3, capacity=cap)
        ids = spade.select(cv, xy_d, point_id_base=3)
        torch.cuda.synchronize()
    finally:
        _set(spade, {})
    opt, opl = oracle.join_pairs(xy, polys, point_id_base=3)
    gpt, gpl = sorted_pairs(pt.cpu().numpy(), pl.cpu().numpy())
    np.testing.assert_array_equal(gpt, opt)
    np.testing.assert_array_equal(gpl, opl)
    np.testing.assert_array_equal(np.sort(ids.cpu().numpy()), oracle.select(xy, polys, point_id_base=3))


def test_split_by_deferral_budget(spade):
    """A boundary-heavy canvas (C1 at 128-unit pixels: nearly every pixel a boundary pixel, so
    the deferral reserves 16 B for about every point) with the smallest deferral budget: the call
    is cut into more sub-launches (more kernel launches), results unchanged."""
    import torch
    polys, xy = _c1_case()
    xy_big = torch.as_tensor(np.tile(xy, (80, 1))).cuda()      # 5M points > 64 MB / 16 B
    expect = 80 * oracle.join_count(xy, polys)
    launches = []
    for budget in (4096, 64):
        _set(spade, {"defer": 1, "defer_budget_mb": budget})
        try:
            cv = spade.Canvas(polys, log2_pixel=7)
            l0 = spade.launch_count()
            counts = spade.join_count(cv, xy_big).cpu().numpy()
            launches.append(spade.launch_count() - l0)
        finally:
            _set(spade, {})
        np.testing.assert_array_equal(counts, expect)
    assert launches[1] > launches[0]


@pytest.mark.slow
def test_count_over_2_31_points_one_call(spade):
    """A real COUNT of n = 2^31 + 13 points in one call (two sub-launches at the default size):
    equal to the sum of two calls below 2^31, and the tiling partition sum(counts) = n."""
    import torch
    w = configs.c3()
    n = (1 << 31) + 13
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    xy = gen.points_device(w.points, w.point_seed, 0, n)
    full = spade.join_count(cv, xy)
    assert int(full.sum()) == n
    parts = torch.zeros_like(full)
    h = n // 2 + 5
    spade.join_count(cv, xy[:h], parts)
    spade.join_count(cv, xy[h:], parts)
    assert torch.equal(full, parts)
    # PAIRS in one call across the seam: one pair per point, ids from the right sub-launch
    pt, pl = spade.join_pairs(cv, xy, point_id_base=5)
    assert pt.numel() == n
    lab = torch.full((n,), -1, dtype=torch.int32, device="cuda")
    lab[pt - 5] = pl
    assert int((lab < 0).sum()) == 0
    assert torch.equal(torch.bincount(pl.long(), minlength=cv.num_polys), full)
    del pt, pl
    seam = (1 << 31) - 64
    idx = np.unique(np.concatenate([np.arange(0, 40), np.arange(seam - 40, seam + 40), np.arange(n - 40, n),
                                    np.random.default_rng(5).integers(0, n, 2000)])).astype(np.int64)
    got = lab[torch.as_tensor(idx, device="cuda")].cpu().numpy().astype(np.int64)
    sub = gen.points_at(w.points, w.point_seed, idx)
    opt, opl = oracle.join_pairs(sub, w.polys)
    exp = np.full(len(idx), -1, np.int64)
    exp[opt] = opl
    np.testing.assert_array_equal(got, exp)


@pytest.mark.slow
@pytest.mark.parametrize("where", ["multi_owner", "boundary_k_agg"])
def test_per_record_counter_never_wraps(spade, where):
    """n = 2^32 + 13 copies of ONE point in one call, on a pixel of two identical squares:
    'multi_owner' = an interior pixel (no edge, owner set {0, 1}: one per-record counter takes
    every point), 'boundary_k_agg' = a boundary pixel whose corner set K = {0, 1} (K aggregation
    forced: one K counter takes every point).  A uint32 counter kept over the whole call would
    end at 13; both polygons must count all n points (34 GB of points)."""
    import torch
    sq = np.array([[0, 0], [1024, 0], [1024, 1024], [0, 1024]], np.int32)
    polys = {"ring_xy": np.concatenate([sq, sq]), "ring_off": np.array([0, 4, 8], np.int64),
             "poly_ring_off": np.array([0, 1, 2], np.int64)}
    p = (500, 500) if where == "multi_owner" else (1, 700)
    n = (1 << 32) + 13
    _set(spade, {"k_agg": 1} if where == "boundary_k_agg" else {})
    try:
        cv = spade.Canvas(polys, log2_pixel=4)
        xy = torch.empty((n, 2), dtype=torch.int32, device="cuda")
        xy[:, 0] = p[0]
        xy[:, 1] = p[1]
        counts = spade.join_count(cv, xy).cpu().numpy()
        del xy
        torch.cuda.empty_cache()
    finally:
        _set(spade, {})
    assert oracle.join_count(np.array([p], np.int32), polys).tolist() == [1, 1]
    assert counts.tolist() == [n, n]
