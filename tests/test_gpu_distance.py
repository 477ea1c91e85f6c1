"""GPU parity of the distance canvas (spade_build_disk_canvas + the probe) against the CPU oracle
(oracle/distance_oracle.c), element by element (-m gpu).

Bar: bit-exact — per-disk counts equal, (point, disk) pair sets equal after sorting, selected id
sets equal.  Inputs seeded and synthetic: random overlapping disks on small lattices at many
canvas resolutions (every pixel class: inside, outside, boundary, multi-owner), points exactly on
disk boundaries (Pythagorean offsets), the Gauss-circle closed form, more than 64 disks in one
pixel (the record slow path), the paper's distance-join workload at reduced and full size.
"""
import numpy as np
import pytest

import gen
import oracle
from gen import configs
from tests.helpers import lattice, sorted_pairs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def spade():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icde_doraiswamyf22_b200 as sp
    sp.load()
    return sp


def _disks(cxy, r2):
    return {"center_xy": np.ascontiguousarray(cxy, np.int32).reshape(-1, 2), "r2": np.asarray(r2, np.int64).reshape(-1)}


def check_disks(sp, disks, xy, s=-1, max_dim=4096, base=0, dense=False):
    import torch
    cv = sp.Canvas.disks(disks["center_xy"], disks["r2"], log2_pixel=s, max_dim=max_dim, dense=dense)
    xy_d = torch.as_tensor(np.ascontiguousarray(xy, np.int32)).cuda()
    counts = sp.join_count(cv, xy_d).cpu().numpy()
    pt, pl = sp.join_pairs(cv, xy_d, point_id_base=base)
    ids = sp.select(cv, xy_d, point_id_base=base)
    torch.cuda.synchronize()
    pt, pl = sorted_pairs(pt.cpu().numpy(), pl.cpu().numpy())
    np.testing.assert_array_equal(counts, oracle.disk_join_count(xy, disks))
    opt, opl = oracle.disk_join_pairs(xy, disks, point_id_base=base)
    np.testing.assert_array_equal(pt, opt)
    np.testing.assert_array_equal(pl, opl)
    np.testing.assert_array_equal(np.sort(ids.cpu().numpy()), oracle.disk_select(xy, disks, point_id_base=base))
    return cv


def boundary_points(disks, per=8, seed=0):
    """Integer points exactly at distance sqrt(r2) (when r2 is a sum of two squares) and just
    inside/outside it, around every disk."""
    rng = np.random.default_rng(seed)
    pts = []
    for (cx, cy), r2 in zip(disks["center_xy"].tolist(), disks["r2"].tolist()):
        R = int(np.floor(np.sqrt(r2)))
        for _ in range(per):
            dx = int(rng.integers(0, R + 1))
            rem = r2 - dx * dx
            dy = int(np.floor(np.sqrt(max(rem, 0))))
            for (u, v) in [(dx, dy), (dx, dy + 1), (dy, dx), (dy + 1, dx)]:
                for sx in (-1, 1):
                    for sy in (-1, 1):
                        pts.append((cx + sx * u, cy + sy * v))
    return np.array(pts, np.int32).reshape(-1, 2)


@pytest.mark.parametrize("seed", range(8))
def test_random_disks_lattice_all_resolutions(spade, seed):
    rng = np.random.default_rng(2000 + seed)
    nd = int(rng.integers(1, 12))
    cxy = rng.integers(0, 48, size=(nd, 2))
    r2 = rng.choice([0, 1, 2, 5, 13, 50, 99, 200, 401, 1000], size=nd)
    if seed % 3 == 0:                     # identical disks (de-duplicated primitives)
        cxy[-1] = cxy[0]; r2[-1] = r2[0]
    disks = _disks(cxy, r2)
    xy = lattice(-40, -40, 90, 90)
    for s in (0, 1, 2, 3, 5, 7):
        check_disks(spade, disks, xy, s=s, dense=bool(seed & 1))


def test_gauss_circle_closed_form_on_gpu(spade):
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "gauss_circle.json")))["r_to_count"]
    rs = sorted(int(r) for r in g)
    disks = _disks([[1000, 1000]] * len(rs), [r * r for r in rs])
    xy = lattice(1000 - 101, 1000 - 101, 1000 + 101, 1000 + 101)
    import torch
    for s in (-1, 0, 2, 4):
        cv = spade.Canvas.disks(disks["center_xy"], disks["r2"], log2_pixel=s)
        counts = spade.join_count(cv, torch.as_tensor(xy).cuda()).cpu().numpy()
        np.testing.assert_array_equal(counts, [g[str(r)] for r in rs])


def test_boundary_points_exact(spade):
    rng = np.random.default_rng(77)
    cxy = rng.integers(10_000, 60_000, size=(40, 2))
    r2 = rng.integers(0, 3_000_000, size=40)
    r2[:5] = [25, 169, 841, 5 ** 2 * 13 ** 2, 65 ** 2]      # sums of two squares
    disks = _disks(cxy, r2)
    xy = boundary_points(disks, per=12)
    for s in (-1, 3, 6, 9):
        check_disks(spade, disks, xy, s=s)


def test_more_than_64_disks_in_a_pixel(spade):
    # 100 concentric disks + 30 coincident ones: records with > 64 distinct disks (slow path)
    c = [[5000, 5000]] * 130
    r2 = list(range(0, 10_000, 100)) + [777] * 30
    disks = _disks(c, r2)
    xy = lattice(4880, 4880, 5120, 5120)
    for s in (4, 6, 8):
        check_disks(spade, disks, xy, s=s)


def test_distance_join_workload_reduced(spade):
    w = configs.dj()
    n = 30_000
    xy = np.concatenate([gen.points_host(w.points, w.point_seed, 0, n), boundary_points(
        {"center_xy": w.disks["center_xy"][:300], "r2": w.disks["r2"][:300]}, per=2)])
    check_disks(spade, w.disks, xy, max_dim=w.max_dim, base=5_000_000_000)


def test_type2_workload_reduced(spade):
    w = configs.dj2()
    xy = gen.points_host(w.points, w.point_seed, 0, 20_000)
    check_disks(spade, w.disks, xy, max_dim=w.max_dim)


def test_disk_argument_errors(spade):
    import torch
    with pytest.raises(spade.SpadeError) as e:
        spade.Canvas.disks([[0, 0]], [-1])
    assert e.value.code == spade.SPADE_ERR_INVALID_ARG
    with pytest.raises(spade.SpadeError) as e:
        spade.Canvas.disks([[2 ** 30 - 10, 0]], [100])          # reaches x = 2^30
    assert e.value.code == spade.SPADE_ERR_COORD_RANGE
    cv = spade.Canvas.disks([[2 ** 30 - 11, -(2 ** 30) + 10]], [100])   # touches the limits: fine
    xy = np.array([[2 ** 30 - 1, -(2 ** 30) + 10], [2 ** 30 - 11, -(2 ** 30)], [2 ** 31 - 1, -(2 ** 31)]], np.int32)
    assert spade.join_count(cv, torch.as_tensor(xy).cuda()).cpu().tolist() == [2]
    empty = spade.Canvas.disks(np.zeros((0, 2), np.int32), np.zeros(0, np.int64))
    assert spade.select(empty, torch.as_tensor(xy).cuda()).numel() == 0


@pytest.mark.slow
def test_distance_join_full_size_sampled(spade):
    """dj at 1e9 points in bench.py's launch configuration: sampled pairs recomputed by the
    oracle point by point, and COUNT == histogram(PAIRS)."""
    import torch
    w = configs.dj()
    n = w.n_points
    cv = spade.Canvas.disks(w.disks["center_xy"], w.disks["r2"], max_dim=w.max_dim)
    xy = gen.points_device(w.points, w.point_seed, 0, n)
    counts = spade.join_count(cv, xy)
    pt, pl = spade.join_pairs(cv, xy)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(torch.bincount(pl.long(), minlength=cv.num_polys).cpu().numpy(), counts.cpu().numpy())
    rng = np.random.default_rng(9)
    idx = np.unique(rng.integers(0, n, 20_000)).astype(np.int64)
    sx = gen.points_at(w.points, w.point_seed, idx)
    opt, opl = oracle.disk_join_pairs(sx, w.disks)
    # GPU pairs of the sampled points
    sel = torch.isin(pt, torch.as_tensor(idx).cuda())
    gpt, gpl = pt[sel].cpu().numpy(), pl[sel].cpu().numpy()
    gpt, gpl = sorted_pairs(gpt, gpl)
    np.testing.assert_array_equal(gpt, idx[opt])
    np.testing.assert_array_equal(gpl, opl)
