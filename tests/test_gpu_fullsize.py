"""GPU parity at BASELINE.json's full sizes, in bench.py's launch configuration (-m gpu).

The oracle cannot join 1e9 points, so full-size runs are checked (a) element by element on
seeded random samples of the outputs, each recomputed by the oracle one point at a time, and
(b) through properties that hold at any size: tilings partition the domain (every point in
exactly one polygon: sum of counts = N, one pair per point), and COUNT equals the histogram of
the PAIRS output of the same points (two different sinks of the probe agree exactly).
"""
import numpy as np
import pytest

import gen
import oracle
from gen import configs

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def sp():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icde_doraiswamyf22_b200 as m
    m.load()
    return m


def _device_points(w, n, start=0):
    return gen.points_device(w.points, w.point_seed, start, n)


def _sample(n, k, seed):
    rng = np.random.default_rng(seed)
    return np.unique(rng.integers(0, n, k)).astype(np.int64)


def _oracle_labels(w, idx):
    """Polygon of each sampled point (-1 = none); asserts <= 1 polygon (tilings)."""
    xy = gen.points_at(w.points, w.point_seed, idx)
    pt, pl = oracle.join_pairs(xy, w.polys)
    assert len(np.unique(pt)) == len(pt)
    lab = np.full(len(idx), -1, np.int64)
    lab[pt] = pl
    return lab


def _labels_from_pairs(pt, pl, n):
    import torch
    lab = torch.full((n,), -1, dtype=torch.int32, device="cuda")
    lab[pt] = pl
    return lab


@pytest.mark.parametrize("cfg,nsample", [("c3", 20000), ("c4", 20000)])
def test_full_size_count_and_pairs(sp, cfg, nsample):
    import torch
    w = getattr(configs, cfg)()
    n = w.n_points
    cv = sp.Canvas(w.polys, max_dim=w.max_dim)
    xy = _device_points(w, n)
    counts = sp.join_count(cv, xy)
    P = cv.num_polys
    assert int(counts.sum()) == n                            # tiling: every point exactly once
    pt, pl = sp.join_pairs(cv, xy)
    assert pt.numel() == n
    assert torch.equal(torch.bincount(pl.long(), minlength=P), counts)   # COUNT == hist(PAIRS)
    lab = _labels_from_pairs(pt, pl, n)
    assert int((lab < 0).sum()) == 0                         # one pair per point, ids 0..n-1
    idx = _sample(n, nsample, 17)
    got = lab[torch.as_tensor(idx, device="cuda")].cpu().numpy().astype(np.int64)
    np.testing.assert_array_equal(got, _oracle_labels(w, idx))


def test_full_size_select_c2(sp):
    import torch
    w = configs.c2()
    n = w.n_points
    cv = sp.Canvas(w.polys, max_dim=w.max_dim)
    xy = _device_points(w, n)
    ids = sp.select(cv, xy, point_id_base=5)
    assert torch.unique(ids).numel() == ids.numel()          # each id once
    mark = torch.zeros(n, dtype=torch.bool, device="cuda")
    mark[ids - 5] = True
    idx = _sample(n, 100000, 23)
    got = mark[torch.as_tensor(idx, device="cuda")].cpu().numpy()
    exp = _oracle_labels(w, idx) >= 0
    np.testing.assert_array_equal(got, exp)
    # COUNT of the 1-polygon canvas equals the selection size
    assert int(sp.join_count(cv, xy)[0]) == ids.numel()


def _boundary_points(polys, k, seed):
    """k points on or next to polygon boundaries: random ring vertices (shared by two or more
    polygons of the tiling: the tie rule decides them), and vertices moved by 1..3 units (within
    the closed pixel the edges touch).  Every one lies in a boundary pixel at any resolution >= 8
    units, so every one takes the exact test."""
    rng = np.random.default_rng(seed)
    v = polys["ring_xy"][rng.integers(0, len(polys["ring_xy"]), k)].astype(np.int64)
    d = rng.integers(-3, 4, (k, 2))
    d[: k // 2] = 0
    return (v + d).astype(np.int32)


def test_full_size_count_c5_one_gpu_shard(sp):
    """Config 5's polygon set (40k zip-code-like tiles) with one GPU's 1B-point shard, plus 6,000
    boundary-pixel points appended (vertices and near-vertex points): COUNT == hist(PAIRS), the
    appended points' labels and 2,000 sampled stream points equal the oracle's."""
    import torch
    w = configs.c5()
    n = w.n_points
    cv = sp.Canvas(w.polys, max_dim=w.max_dim)
    nb = 6000
    bxy = _boundary_points(w.polys, nb, 41)
    xy = torch.empty((n + nb, 2), dtype=torch.int32, device="cuda")
    gen.points_device(w.points, w.point_seed, 3 * n, n, out=xy[:n])   # shard 3 of 8: global ids [3n, 4n)
    xy[n:] = torch.as_tensor(bxy, device="cuda")
    counts = sp.join_count(cv, xy)
    pt, pl = sp.join_pairs(cv, xy, point_id_base=3 * n)
    assert torch.equal(torch.bincount(pl.long(), minlength=cv.num_polys), counts)
    lab = _labels_from_pairs(pt - 3 * n, pl, n + nb)
    assert int((lab[:n] < 0).sum()) == 0                       # the stream lies inside the tiling
    idx = _sample(n, 2000, 29)
    got = lab[torch.as_tensor(idx, device="cuda")].cpu().numpy().astype(np.int64)
    np.testing.assert_array_equal(got, _oracle_labels(w, idx + 3 * n))
    bpt, bpl = oracle.join_pairs(bxy, w.polys)
    assert len(np.unique(bpt)) == len(bpt)
    exp = np.full(nb, -1, np.int64)
    exp[bpt] = bpl
    np.testing.assert_array_equal(lab[n:].cpu().numpy().astype(np.int64), exp)


def test_full_size_overlap_heavy_ov(sp):
    """NEXT(4)'s scenario: 1,000 overlapping stars (~32 polygons per point on average).  COUNT of
    a 50M-point slice equals the histogram of its PAIRS output; sampled points' pairs equal the
    oracle's; COUNT over the full 1B points equals the sum of its 50M-point slices."""
    import torch
    w = configs.ov()
    n = w.n_points
    cv = sp.Canvas(w.polys, max_dim=w.max_dim)
    m = 50_000_000
    xy = _device_points(w, m, start=7 * m)
    counts = sp.join_count(cv, xy)
    pt, pl = sp.join_pairs(cv, xy, point_id_base=7 * m, capacity=int(counts.sum()))
    assert len(pt) == int(counts.sum())
    assert torch.equal(torch.bincount(pl.long(), minlength=cv.num_polys), counts)
    idx = _sample(m, 200, 31)
    o = torch.argsort(pt)
    pts, pls = pt[o], pl[o]
    lo = torch.searchsorted(pts, torch.as_tensor(idx + 7 * m, device="cuda"))
    hi = torch.searchsorted(pts, torch.as_tensor(idx + 7 * m, device="cuda"), right=True)
    xs = gen.points_at(w.points, w.point_seed, idx + 7 * m)
    opt, opl = oracle.join_pairs(xs, w.polys)
    lo, hi = lo.cpu().numpy(), hi.cpu().numpy()
    for k in range(len(idx)):
        got = np.sort(pls[lo[k]:hi[k]].cpu().numpy().astype(np.int64))
        np.testing.assert_array_equal(got, np.sort(opl[opt == k]))
    del pt, pl, pts, pls, o
    total = torch.zeros(cv.num_polys, dtype=torch.int64, device="cuda")
    full = torch.zeros(cv.num_polys, dtype=torch.int64, device="cuda")
    for s in range(0, n, 200_000_000):
        xs_d = _device_points(w, min(200_000_000, n - s), start=s)
        sp.join_count(cv, xs_d, total)
        del xs_d
    xy_full = _device_points(w, n)
    sp.join_count(cv, xy_full, full)
    assert torch.equal(total, full)
