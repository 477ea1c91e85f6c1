"""GPU parity of kNN selection (spade_knn and its three steps) against the CPU oracle
(oracle.knn: sort every point by (dist2, id), keep k) — bit-exact ids and squared distances.

The circle aggregation of step 1 is checked against the distance oracle: COUNT(circle b) must
equal oracle.disk_join_count over the concentric disks of radius^2 = r2_b (the bucket upper ends,
include/spade.h).  Full size: 1e9 points in bench.py's configuration, checked by properties
(order, recomputed distances, separation against a large random sample, and the disk canvas
counting the same circles).
"""
import numpy as np
import pytest

import gen
import oracle
from gen import configs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def spade():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icde_doraiswamyf22_b200 as sp
    sp.load()
    return sp


def bucket_r2(b):
    """Squared radius of circle b (include/spade.h, SPADE_KNN_BINS)."""
    if b < 4:
        return b
    e, j = 2 + (b - 4) // 4, (b - 4) % 4
    return (1 << e) + (j + 1) * (1 << (e - 2)) - 1


def _check(sp, xy, q, k, base=0):
    import torch
    ids, d2 = sp.knn(torch.as_tensor(xy).cuda(), q, k, point_id_base=base)
    oids, od2 = oracle.knn(xy, q, k, point_id_base=base)
    np.testing.assert_array_equal(ids.cpu().numpy(), oids)
    np.testing.assert_array_equal(d2.cpu().numpy(), od2)


@pytest.mark.parametrize("seed", range(6))
def test_knn_random_matches_oracle(spade, seed):
    rng = np.random.default_rng(300 + seed)
    n = int(rng.integers(1, 50_000))
    span = int(rng.choice([8, 100, 10_000, 1 << 24]))
    xy = rng.integers(-span, span, size=(n, 2)).astype(np.int32)
    q = tuple(int(v) for v in rng.integers(-span, span, 2))
    for k in (1, 2, 7, 50, 1000, n, n + 5):
        _check(spade, xy, q, k, base=int(rng.integers(0, 1 << 40)))


def test_knn_ties_and_duplicates(spade):
    # lattice around q: many equal distances; duplicates of the same point
    xs, ys = np.meshgrid(np.arange(-20, 21), np.arange(-20, 21))
    xy = np.stack([xs.ravel(), ys.ravel()], 1).astype(np.int32)
    xy = np.concatenate([xy, xy[::7], xy[::13]])
    xy = xy[np.random.default_rng(1).permutation(len(xy))]
    for k in range(0, 120, 7):
        _check(spade, xy, (0, 0), k)
    _check(spade, xy, (3, -2), 333)


def test_knn_extreme_coordinates(spade):
    lo, hi = -(1 << 30), (1 << 30) - 1
    xy = np.array([[lo, lo], [hi, hi], [lo, hi], [hi, lo], [0, 0], [hi, hi]], np.int32)
    for q in [(lo, lo), (hi, hi), (0, 0), (lo, hi)]:
        for k in (1, 3, 6):
            _check(spade, xy, q, k)


def test_circle_aggregation_matches_disk_oracle(spade):
    import torch
    w = configs.knn()
    xy = gen.points_host(w.points, w.point_seed, 0, 200_000)
    q = w.query
    hist = spade.knn_histogram(torch.as_tensor(xy).cuda(), q).cpu().numpy()
    assert hist[-1] == 0 and hist[:-1].sum() == len(xy)
    bs = np.array([0, 1, 3, 4, 10, 40, 80, 100, 120, 140, 160, 200, 247])
    r2 = np.array([bucket_r2(int(b)) for b in bs], np.int64)
    disks = {"center_xy": np.tile(np.array([q], np.int32), (len(bs), 1)), "r2": r2}
    np.testing.assert_array_equal(np.cumsum(hist[:-1])[bs], oracle.disk_join_count(xy, disks))
    # and the distance canvas (an independent GPU path) counts the same circles
    r2c = r2[r2 < (1 << 46)]
    ok = (q[0] - np.floor(np.sqrt(r2c)) >= -(1 << 30))
    cv = spade.Canvas.disks(np.tile(np.array([q], np.int32), (int(ok.sum()), 1)), r2c[ok])
    np.testing.assert_array_equal(spade.join_count(cv, torch.as_tensor(xy).cuda()).cpu().numpy(),
                                  np.cumsum(hist[:-1])[bs][: len(r2c)][ok])


def test_knn_steps_compose(spade):
    import torch
    rng = np.random.default_rng(5)
    xy = rng.integers(0, 1 << 20, size=(100_000, 2)).astype(np.int32)
    q, k = (500_000, 400_000), 321
    xd = torch.as_tensor(xy).cuda()
    h = spade.knn_histogram(xd, q).cpu().numpy()
    r2, cnt = spade.knn_radius(h, k)
    assert cnt >= k and int((((xy.astype(np.int64) - q) ** 2).sum(1) <= r2).sum()) == cnt
    ids, d2 = spade.knn_select(xd, q, r2)
    assert ids.numel() == cnt
    ti, td = spade.knn_topk(ids, d2, k)
    oi, od = oracle.knn(xy, q, k)
    np.testing.assert_array_equal(ti.cpu().numpy(), oi)
    np.testing.assert_array_equal(td.cpu().numpy(), od)


def test_knn_errors(spade):
    import torch
    xy = torch.as_tensor(np.array([[0, 0], [1 << 30, 0]], np.int32)).cuda()
    with pytest.raises(spade.SpadeError) as e:
        spade.knn(xy, (0, 0), 1)
    assert e.value.code == spade.SPADE_ERR_COORD_RANGE
    with pytest.raises(spade.SpadeError) as e:
        spade.knn(xy[:1], (1 << 30, 0), 1)
    assert e.value.code == spade.SPADE_ERR_COORD_RANGE
    ids, d2 = spade.knn(xy[:1], (0, 0), 0)
    assert ids.numel() == 0
    ids, d2 = spade.knn(xy[:0], (0, 0), 5)
    assert ids.numel() == 0


@pytest.mark.slow
def test_knn_full_size(spade):
    import torch
    w = configs.knn()
    n = w.n_points
    xy = gen.points_device(w.points, w.point_seed, 0, n)
    ids, d2 = spade.knn(xy, w.query, w.k)
    ids, d2 = ids.cpu().numpy(), d2.cpu().numpy()
    assert len(ids) == w.k
    key = list(zip(d2.tolist(), ids.tolist()))
    assert key == sorted(key)
    pts = gen.points_at(w.points, w.point_seed, ids).astype(np.int64)
    np.testing.assert_array_equal(((pts - np.array(w.query)) ** 2).sum(1), d2)
    # separation against a large random sample: nothing outside the result is closer
    idx = np.unique(np.random.default_rng(4).integers(0, n, 2_000_000)).astype(np.int64)
    sp_ = gen.points_at(w.points, w.point_seed, idx).astype(np.int64)
    sd = ((sp_ - np.array(w.query)) ** 2).sum(1)
    outside = ~np.isin(idx, ids)
    kd, kid = key[-1]
    assert np.all((sd[outside] > kd) | ((sd[outside] == kd) & (idx[outside] > kid)))
    # the distance canvas counts exactly k points within d2_k when there is no tie at the k-th
    cv = spade.Canvas.disks(np.array([w.query], np.int32), [kd])
    c = int(spade.join_count(cv, xy).cpu()[0])
    assert c >= w.k
    cv2 = spade.Canvas.disks(np.array([w.query], np.int32), [kd - 1])
    assert int(spade.join_count(cv2, xy).cpu()[0]) < w.k
