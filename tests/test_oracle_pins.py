"""Pins of the CPU oracle to things OTHER than itself (-m "not gpu").

The paper prints no worked example (Fig. 4, is an image), so the oracle is
pinned by: hand-derived golden cases (tests/golden/hand_cases.json), an independent tie-free
textbook test at a symbolically perturbed point, the winding number on simple polygons, closed
forms (rectangle lattice counts, grid tilings), independent labelings (kd-descent over guillotine
parcels), invariants (tilings partition the plane, hole + island = outer, chord splits) and
metamorphic relations (translation, integer scaling, orientation, start vertex).  Each is chosen
so that a plausible slip in the oracle (a dropped closing edge, a flipped comparison, o >= 0 vs
o > 0, a transposed product, a lost ring) fails at least one of them.
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import gen
import oracle
from gen import polygons as pg
from tests.helpers import lattice, random_polyset

HERE = os.path.dirname(os.path.abspath(__file__))


def _one(rings):
    return pg.assemble([[np.asarray(r) for r in rings]])


def _inside_set(polys, xy, p=0):
    pt, pl = oracle.join_pairs(xy, polys)
    return set(pt[pl == p].tolist())


# --------------------------------------------------------------------------------------------
# 1. hand-derived golden cases (tie rule, holes, degenerate and self-intersecting rings)

GOLDEN = json.load(open(os.path.join(HERE, "golden", "hand_cases.json")))["cases"]


@pytest.mark.parametrize("case", GOLDEN, ids=[c["name"] for c in GOLDEN])
def test_golden_hand_cases(case):
    polys = _one(case["rings"])
    x0, y0, x1, y1 = case["box"]
    xy = lattice(x0, y0, x1, y1)
    ids = oracle.select(xy, polys)
    got = sorted(map(tuple, xy[ids].tolist()))
    assert got == sorted(map(tuple, case["inside"]))
    # the per-point entry point agrees with the batch one
    for (x, y) in xy[:: max(1, len(xy) // 17)].tolist():
        assert oracle.point_in_polygon(x, y, polys, 0) == ((x, y) in set(got))


# --------------------------------------------------------------------------------------------
# 2. tie rule == strict textbook crossing test at the perturbed point M*p + (k, 1)
#    (k > D, M > D(k+1); no ties can occur there, asserted below)

def _strict_inside(rings, qx, qy):
    """Textbook crossing number with exact rationals; ASSERTS no degenerate configuration."""
    inside = False
    for r in rings:
        n = len(r)
        for i in range(n):
            ax, ay = r[i]; bx, by = r[(i + 1) % n]
            assert ay != qy and by != qy, "tie: vertex at the ray's height"
            if (ay > qy) != (by > qy):
                xc = Fraction(ax) + Fraction((bx - ax) * (qy - ay), by - ay)
                assert xc != qx, "tie: point on an edge"
                if xc > qx:
                    inside = not inside
    return inside


@pytest.mark.parametrize("seed", range(8))
def test_half_open_rule_equals_perturbed_strict_test(seed):
    rng = np.random.default_rng(seed)
    polys = random_polyset(rng, 0, 9, 3)
    xy = lattice(-1, -1, 10, 10)
    D = 12
    k = D + 1
    M = D * (k + 1) + 1
    pt, pl = oracle.join_pairs(xy, polys)
    got = set(zip(pt.tolist(), pl.tolist()))
    for p, rings in enumerate(pg.polygons_as_lists(polys)):
        srings = [[(int(x) * M, int(y) * M) for x, y in r.tolist()] for r in rings]
        for i, (x, y) in enumerate(xy.tolist()):
            assert _strict_inside(srings, M * x + k, M * y + 1) == ((i, p) in got), (p, x, y)


# --------------------------------------------------------------------------------------------
# 3. simple polygons, points off the boundary: winding number != 0  (Sunday's algorithm)

def _winding(ring, px, py):
    wn = 0
    n = len(ring)
    for i in range(n):
        ax, ay = ring[i]; bx, by = ring[(i + 1) % n]
        is_left = (bx - ax) * (py - ay) - (px - ax) * (by - ay)
        if ay <= py < by and is_left > 0:
            wn += 1
        elif by <= py < ay and is_left < 0:
            wn -= 1
    return wn


def _on_boundary(ring, px, py):
    n = len(ring)
    for i in range(n):
        ax, ay = ring[i]; bx, by = ring[(i + 1) % n]
        if (bx - ax) * (py - ay) == (by - ay) * (px - ax) and min(ax, bx) <= px <= max(ax, bx) \
                and min(ay, by) <= py <= max(ay, by):
            return True
    return False


@pytest.mark.parametrize("seed", range(6))
def test_winding_number_on_simple_polygons(seed):
    rng = np.random.default_rng(100 + seed)
    rings = [pg.star(rng, int(rng.integers(5, 30)), 500, 500, 400, 300, rmin=0.6),
             pg.convex_hull(rng.integers(0, 1000, (30, 2)))]
    xy = rng.integers(-50, 1050, (3000, 2)).astype(np.int32)
    for ring in rings:
        polys = _one([ring])
        ins = _inside_set(polys, xy)
        r = ring.tolist()
        for i, (x, y) in enumerate(xy.tolist()):
            if _on_boundary(r, x, y):
                continue
            assert (_winding(r, x, y) != 0) == (i in ins)


# --------------------------------------------------------------------------------------------
# 4. closed forms

@pytest.mark.parametrize("seed", range(5))
def test_rectangle_lattice_count_closed_form(seed):
    rng = np.random.default_rng(200 + seed)
    rects = []
    for _ in range(20):
        x0, x1 = sorted(rng.integers(-30, 30, 2)); y0, y1 = sorted(rng.integers(-30, 30, 2))
        rects.append((int(x0), int(y0), int(x1), int(y1)))
    polys = pg.assemble([[pg.rect(*r) if i % 2 else pg.rect(*r)[::-1]] for i, r in enumerate(rects)])
    counts = oracle.join_count(lattice(-35, -35, 35, 35), polys)
    assert counts.tolist() == [(x1 - x0) * (y1 - y0) for (x0, y0, x1, y1) in rects]


def test_grid_tiling_counts_closed_form():
    polys = pg.grid_tiling(4, 4, 0, 0, 256, 256)
    xy = gen.points_host(gen.uniform_params(0, 0, 1024, 1024), 3, 0, 20000)
    counts = oracle.join_count(xy, polys)
    expect = np.bincount((xy[:, 1] >> 8) * 4 + (xy[:, 0] >> 8), minlength=16)
    assert counts.tolist() == expect.tolist()


def test_guillotine_parcels_match_kd_labels():
    """Non-intersecting rectangle parcels: labels by kd-descent, no PIP arithmetic."""
    rng = np.random.default_rng(7)
    rects, tree = pg.guillotine_parcels(rng, 300, 0, 0, 4000, 3000)
    polys = pg.assemble([[pg.rect(*r)] for r in rects])
    xy = np.concatenate([gen.points_host(gen.uniform_params(0, 0, 4000, 3000), 11, 0, 5000),
                         np.array([[r[0], r[1]] for r in rects] + [[r[2] - 1, r[3] - 1] for r in rects], np.int32)])
    pt, pl = oracle.join_pairs(xy, polys)
    assert pt.tolist() == list(range(len(xy)))                      # exactly one parcel each
    assert pl.tolist() == [pg.kd_label(tree, int(x), int(y)) for x, y in xy.tolist()]


# --------------------------------------------------------------------------------------------
# 5. invariants

def test_jittered_tiling_with_islands_is_a_partition():
    polys = pg.jittered_tiling(5, 4, 12, domain=1 << 16, n_islands=3, seed=3)
    xy = np.concatenate([gen.points_host(gen.uniform_params(0, 0, 1 << 16, 1 << 16), 5, 0, 20000),
                         polys["ring_xy"][::7]])                      # plus points ON shared borders
    pt, pl = oracle.join_pairs(xy, polys)
    inside_domain = (xy[:, 0] < (1 << 16)) & (xy[:, 1] < (1 << 16))
    assert pt.tolist() == np.nonzero(inside_domain)[0].tolist()      # one polygon per point
    # points outside the canvas extent join nothing (P:182 clipping)
    far = np.array([[-1, 5], [5, -1], [1 << 16, 3], [3, 1 << 16], [-(2**31), 2**31 - 1]], np.int32)
    assert oracle.join_count(far, polys).sum() == 0


def test_hole_plus_island_equals_outer():
    rng = np.random.default_rng(11)
    outer = pg.star(rng, 40, 500, 500, 450, 450, rmin=0.8)
    hole = pg.star(rng, 25, 500, 500, 200, 200, rmin=0.7)
    xy = np.concatenate([lattice(0, 0, 1000, 1000)[::3], outer, hole]).astype(np.int32)
    holed = pg.assemble([[outer, hole[::-1]], [hole]])
    c = oracle.join_pairs(xy, holed)
    ins = set(c[0].tolist())
    assert len(c[0]) == len(ins)                                      # never in both
    alone = _inside_set(_one([outer]), xy)
    assert ins == alone


@pytest.mark.parametrize("seed", range(4))
def test_chord_split_is_xor_additive(seed):
    rng = np.random.default_rng(300 + seed)
    ring = pg.star(rng, 24, 100, 100, 90, 90, rmin=0.3)
    i, k = 3, 15
    a = np.concatenate([ring[i:k + 1]])
    b = np.concatenate([ring[k:], ring[:i + 1]])
    xy = lattice(0, 0, 200, 200)
    whole = _inside_set(_one([ring]), xy)
    sa, sb = _inside_set(_one([a]), xy), _inside_set(_one([b]), xy)
    assert whole == sa ^ sb
    # a convex polygon split by a chord: the halves partition it (SUM-additive)
    hull = pg.convex_hull(rng.integers(0, 200, (40, 2)))
    h1, h2 = hull[: len(hull) // 2 + 1], np.concatenate([hull[len(hull) // 2:], hull[:1]])
    c = oracle.join_count(xy, pg.assemble([[hull], [h1], [h2]]))
    assert c[0] == c[1] + c[2]


# --------------------------------------------------------------------------------------------
# 6. metamorphic relations

@pytest.mark.parametrize("seed", range(4))
def test_translation_scaling_orientation_start_invariance(seed):
    rng = np.random.default_rng(400 + seed)
    polys = random_polyset(rng, 0, 30, 4)
    xy = lattice(-2, -2, 32, 32)
    base = oracle.join_pairs(xy, polys)
    lists = pg.polygons_as_lists(polys)
    tx, ty, sc = int(rng.integers(-10**6, 10**6)), int(rng.integers(-10**6, 10**6)), int(rng.integers(2, 50))
    moved = pg.assemble([[r * sc + np.array([tx, ty]) for r in rs] for rs in lists])
    got = oracle.join_pairs(xy.astype(np.int64) * sc + np.array([tx, ty]), moved)
    assert all(np.array_equal(u, v) for u, v in zip(base, got))
    flipped = pg.assemble([[np.roll(r[::-1], int(rng.integers(0, len(r))), axis=0) for r in rs] for rs in lists])
    got = oracle.join_pairs(xy, flipped)
    assert all(np.array_equal(u, v) for u, v in zip(base, got))


def test_select_pairs_count_agree():
    w_polys = pg.c1_polygons(102)
    xy = gen.points_host(gen.uniform_params(0, 0, 1024, 1024), 101, 0, 5000)
    pt, pl = oracle.join_pairs(xy, w_polys, point_id_base=77)
    counts = oracle.join_count(xy, w_polys)
    ids = oracle.select(xy, w_polys, point_id_base=77)
    assert np.bincount(pl, minlength=len(counts)).tolist() == counts.tolist()
    assert ids.tolist() == sorted(set(pt.tolist()))
    assert counts.sum() > len(ids) > 0          # config 1 overlaps: some points in >1 polygon


# --------------------------------------------------------------------------------------------
# 7. the R-tree CPU baseline agrees with the brute-force oracle

@pytest.mark.parametrize("seed", range(3))
def test_rtree_baseline_matches_oracle(seed):
    rng = np.random.default_rng(500 + seed)
    polys = random_polyset(rng, 0, 60, 12)
    xy = lattice(-3, -3, 63, 63)
    assert oracle.rtree_join_count(xy, polys).tolist() == oracle.join_count(xy, polys).tolist()
    t = pg.jittered_tiling(7, 5, 20, domain=1 << 18, n_islands=3, seed=seed)
    xy2 = gen.points_host(gen.taxi_params(seed, domain=1 << 18), seed, 0, 20000)
    assert oracle.rtree_join_count(xy2, t).tolist() == oracle.join_count(xy2, t).tolist()
