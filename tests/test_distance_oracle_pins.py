"""Pins of the distance/kNN oracle (oracle/distance_oracle.c) to things OTHER than itself
(-m "not gpu").

PAPER.md prints no worked distance example, so the closed-disk predicate is
pinned by: published lattice counts of the Gauss circle problem (tests/golden/gauss_circle.json),
Jacobi's two-square theorem (r_2(k) = 4 (d_1(k) - d_3(k)), a divisor count that shares no
arithmetic with the distance test), Pythagorean boundary points (closed disk), the dihedral
symmetry of a disk about its centre, translation invariance, and exact arithmetic near the
coordinate limits.  kNN is pinned by the lattice: the k = N(r) nearest lattice points to
the centre are exactly the lattice points of the disk, and by the prefix / separation invariants.
Each is chosen so that a plausible slip (< for <=, a dropped or doubled term, a swapped axis, an
int64 overflow, an unstable tie order) fails at least one of them.
"""
import json
import os

import numpy as np
import pytest

import oracle
from tests.helpers import lattice

HERE = os.path.dirname(os.path.abspath(__file__))
GAUSS = json.load(open(os.path.join(HERE, "golden", "gauss_circle.json")))["r_to_count"]


def _disk(cx, cy, r2):
    return {"center_xy": np.array([[cx, cy]], np.int32), "r2": np.array([r2], np.int64)}


def _jacobi_N(n):
    """1 + sum_{k=1..n} r_2(k),  r_2(k) = 4 (#divisors = 1 mod 4  -  #divisors = 3 mod 4)."""
    tot = 1
    for k in range(1, n + 1):
        d1 = d3 = 0
        for d in range(1, k + 1, 2):
            if k % d == 0:
                if d % 4 == 1:
                    d1 += 1
                else:
                    d3 += 1
        tot += 4 * (d1 - d3)
    return tot


@pytest.mark.parametrize("r", sorted(int(r) for r in GAUSS))
def test_gauss_circle_published_counts(r):
    xy = lattice(-r - 1, -r - 1, r + 1, r + 1)
    assert int(oracle.disk_join_count(xy, _disk(0, 0, r * r))[0]) == GAUSS[str(r)]


def test_jacobi_two_square_closed_form():
    # every integer squared radius 0..300 (most are not perfect squares), off-origin centre
    cx, cy = 1234, -777
    xy = lattice(cx - 18, cy - 18, cx + 18, cy + 18)
    r2s = np.arange(0, 301, dtype=np.int64)
    disks = {"center_xy": np.tile(np.array([[cx, cy]], np.int32), (len(r2s), 1)), "r2": r2s}
    got = oracle.disk_join_count(xy, disks)
    want = np.array([_jacobi_N(int(n)) for n in r2s])
    np.testing.assert_array_equal(got, want)


def test_closed_boundary_pythagorean():
    # (3,4,5), (5,12,13), (20,21,29): points exactly at distance r are inside; r^2 - 1 excludes them
    for a, b, c in [(3, 4, 5), (5, 12, 13), (20, 21, 29)]:
        for sx in (-1, 1):
            for sy in (-1, 1):
                assert oracle.in_disk(7 + sx * a, -3 + sy * b, 7, -3, c * c)
                assert not oracle.in_disk(7 + sx * a, -3 + sy * b, 7, -3, c * c - 1)
                assert oracle.in_disk(7 + sy * b, -3 + sx * a, 7, -3, c * c)
    assert oracle.in_disk(5, 5, 5, 5, 0) and not oracle.in_disk(5, 6, 5, 5, 0)


def test_dihedral_symmetry_and_translation():
    rng = np.random.default_rng(11)
    cx, cy, r2 = 100, -50, 1000
    pts = rng.integers(-60, 61, size=(3000, 2))
    base = np.array([oracle.in_disk(cx + u, cy + v, cx, cy, r2) for u, v in pts.tolist()])
    for f in (lambda u, v: (-v, u), lambda u, v: (u, -v), lambda u, v: (v, u), lambda u, v: (-u, -v)):
        img = np.array([oracle.in_disk(cx + f(u, v)[0], cy + f(u, v)[1], cx, cy, r2) for u, v in pts.tolist()])
        np.testing.assert_array_equal(base, img)
    shifted = np.array([oracle.in_disk(cx + u + 999, cy + v - 4242, cx + 999, cy - 4242, r2) for u, v in pts.tolist()])
    np.testing.assert_array_equal(base, shifted)
    # and it is not a square / diamond: both the corner and the axis extreme are decided correctly
    assert oracle.in_disk(cx + 31, cy, cx, cy, r2) and not oracle.in_disk(cx + 32, cy, cx, cy, r2)
    assert oracle.in_disk(cx + 22, cy + 22, cx, cy, r2) and not oracle.in_disk(cx + 23, cy + 22, cx, cy, r2)


def test_exact_near_coordinate_limits():
    # |dx|, |dy| up to 2^31 - 1: the squares reach 2^62 and their sum ~2^63 (overflows int64 sums)
    lo, hi = -(2 ** 30), 2 ** 30 - 1
    for (px, py, cx, cy) in [(lo, lo, hi, hi), (hi, lo, lo, hi), (lo, 0, hi, 0), (lo, hi, hi, lo + 5)]:
        d2 = (px - cx) ** 2 + (py - cy) ** 2
        assert d2 < 2 ** 63
        assert oracle.in_disk(px, py, cx, cy, d2)
        assert not oracle.in_disk(px, py, cx, cy, d2 - 1)
    # points are any int32: |dx| up to 3 * 2^30, dx^2 ~ 9 * 2^60 > 2^63 (no disk reaches them)
    for (px, py, cx, cy) in [(-(2 ** 31), 0, hi, 0), (-(2 ** 31), 2 ** 31 - 1, hi, lo), (2 ** 31 - 1, -(2 ** 31), lo, hi)]:
        assert (px - cx) ** 2 > 2 ** 63
        assert not oracle.in_disk(px, py, cx, cy, 2 ** 63 - 1)


def test_join_ops_consistent_and_type1_equals_type2():
    rng = np.random.default_rng(5)
    xy = rng.integers(0, 200, size=(4000, 2)).astype(np.int32)
    cxy = rng.integers(0, 200, size=(25, 2)).astype(np.int32)
    r2 = np.full(25, 400, np.int64)
    d = {"center_xy": cxy, "r2": r2}
    counts = oracle.disk_join_count(xy, d)
    pt, pl = oracle.disk_join_pairs(xy, d)
    np.testing.assert_array_equal(np.bincount(pl, minlength=25), counts)
    np.testing.assert_array_equal(oracle.disk_select(xy, d), np.unique(pt))
    # type 2 with equal radii == type 1; per-disk radii change only their own disk's count
    r2b = r2.copy(); r2b[3] = 0
    c2 = oracle.disk_join_count(xy, {"center_xy": cxy, "r2": r2b})
    np.testing.assert_array_equal(np.delete(c2, 3), np.delete(counts, 3))
    assert c2[3] == int(((xy[:, 0] == cxy[3, 0]) & (xy[:, 1] == cxy[3, 1])).sum())
    # pairs sorted by (point, disk) and offset by the id base
    pt2, pl2 = oracle.disk_join_pairs(xy, d, point_id_base=10 ** 12)
    np.testing.assert_array_equal(pt2 - 10 ** 12, pt)
    assert np.all(np.diff(pt) >= 0)


def test_knn_lattice_equals_disk():
    # the N(r) nearest lattice points to the centre are the disk's lattice points (no ties cut)
    xy = lattice(-12, -12, 12, 12)
    rng = np.random.default_rng(3)
    xy = xy[rng.permutation(len(xy))]
    for r in range(0, 11):
        k = GAUSS[str(r)]
        ids, d2 = oracle.knn(xy, (0, 0), k)
        inside = {i for i, (x, y) in enumerate(xy.tolist()) if x * x + y * y <= r * r}
        assert set(ids.tolist()) == inside
        assert int(d2.max()) <= r * r


def test_knn_order_prefix_and_ties():
    rng = np.random.default_rng(8)
    xy = rng.integers(-50, 50, size=(2000, 2)).astype(np.int32)
    q = (3, -7)
    ids_all, d2_all = oracle.knn(xy, q, 10 ** 9)
    assert len(ids_all) == len(xy) and sorted(ids_all.tolist()) == list(range(len(xy)))
    key = list(zip(d2_all.tolist(), ids_all.tolist()))
    assert key == sorted(key)                                   # (dist2, id) order, ties by id
    for k in (0, 1, 7, 100, 1999):
        ids, d2 = oracle.knn(xy, q, k)
        np.testing.assert_array_equal(ids, ids_all[:k])
    # separation: every unselected point is at least as far as the k-th
    ids, d2 = oracle.knn(xy, q, 100)
    rest = np.setdiff1d(np.arange(len(xy)), ids)
    dr = (xy[rest, 0].astype(np.int64) - q[0]) ** 2 + (xy[rest, 1].astype(np.int64) - q[1]) ** 2
    assert dr.min() >= d2.max()
    ids_b, _ = oracle.knn(xy, q, 100, point_id_base=500)
    np.testing.assert_array_equal(ids_b - 500, ids)
