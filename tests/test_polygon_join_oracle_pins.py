"""Pins of the polygon x polygon join oracle (oracle/polygon_join_oracle.c; -m "not gpu").

The oracle decides ST_INTERSECTS of closed regions (reading C15)
by closed-segment contact or ring-vertex containment.  It is pinned to things other than itself:
  * hand-derived cases (tests/golden/polygon_join_cases.json);
  * the textbook segment test on hand cases (collinear overlaps, touching endpoints, crossings);
  * a closed form: a k x m grid of touching rectangles, self-joined, pairs = cells at Chebyshev
    distance <= 1 (shared sides and shared corners);
  * lattice witnesses: a lattice point in both closed regions (inside by the half-open rule of the
    point oracle, or on an edge by an exact collinearity test) forces "intersect", and disjointness
    is cross-checked on a 4x finer lattice;
  * invariants of the closed predicate: symmetry, integer translation and scaling, ring
    orientation and start vertex, and the 90-degree rotations and reflections (which the
    half-open POINT rule does not have: the oracle only uses it away from every edge, where it
    equals the strict test).
"""
import json
import os

import numpy as np
import pytest

import oracle
from gen import polygons as pg
from tests.helpers import valid_polyset as _valid_polyset

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CASES = json.load(open(os.path.join(ROOT, "tests", "golden", "polygon_join_cases.json")))["cases"]


def _one(rings):
    return pg.assemble([[np.array(r, np.int64) for r in rings]])


@pytest.mark.parametrize("case", CASES, ids=lambda c: c["name"])
def test_hand_cases(case):
    A, B = _one(case["A"]), _one(case["B"])
    assert oracle.polygons_intersect(A, 0, B, 0) == case["expect"], case["why"]
    assert oracle.polygons_intersect(B, 0, A, 0) == case["expect"]          # symmetric
    a, b = oracle.polygon_join(A, B)
    assert (len(a) == 1) == case["expect"]


def test_segment_hand_cases():
    si = oracle.segments_intersect
    assert si((0, 0), (4, 4), (0, 4), (4, 0))            # proper crossing at (2, 2)
    assert si((0, 0), (4, 4), (2, 2), (9, 0))            # endpoint on the other segment
    assert si((0, 0), (4, 0), (4, 0), (9, 3))            # shared endpoint
    assert si((0, 0), (4, 0), (2, 0), (9, 0))            # collinear overlap
    assert not si((0, 0), (4, 0), (5, 0), (9, 0))        # collinear, disjoint
    assert not si((0, 0), (4, 4), (1, 0), (5, 4))        # parallel
    assert not si((0, 0), (4, 4), (3, 0), (9, -6))       # lines cross outside both segments
    assert not si((0, 0), (1, 3), (1, 2), (5, 2))        # near miss: (1, 3)-(0, 0) passes x = 2/3 at y = 2
    assert si((0, 0), (3, 3), (3, 3), (3, 3))            # degenerate point on the segment end


def test_grid_tiling_closed_form():
    k, m = 5, 4
    polys = pg.grid_tiling(k, m, 0, 0, 100, 70)
    a, b = oracle.polygon_join(polys, polys)
    got = set(zip(a.tolist(), b.tolist()))
    exp = {(j1 * k + i1, j2 * k + i2) for j1 in range(m) for i1 in range(k) for j2 in range(m) for i2 in range(k)
           if abs(i1 - i2) <= 1 and abs(j1 - j2) <= 1}
    assert got == exp


def test_grid_vs_shifted_grid_closed_form():
    """Rectangles [100i, 100i+100] x [70j, 70j+70] against the same grid shifted by (+50, +35):
    cell (i, j) meets shifted cell (i', j') iff its x-range [100i, 100i+100] meets
    [100i'+50, 100i'+150] (i' in {i-1, i}) and likewise for y."""
    k, m = 4, 3
    A = pg.grid_tiling(k, m, 0, 0, 100, 70)
    B = pg.grid_tiling(k, m, 50, 35, 100, 70)
    a, b = oracle.polygon_join(A, B)
    exp = {(j * k + i, j2 * k + i2) for j in range(m) for i in range(k) for j2 in range(m) for i2 in range(k)
           if i2 in (i - 1, i) and j2 in (j - 1, j)}
    assert set(zip(a.tolist(), b.tolist())) == exp


def _closed_member(xy, polys, p):
    """Lattice points in the CLOSED region of polygon p: half-open inside (point oracle) or on an
    edge (exact collinearity + bounding box; independent of the join oracle)."""
    xy = np.asarray(xy, np.int64)
    inside = np.array([oracle.point_in_polygon(int(x), int(y), polys, p) for x, y in xy], bool)
    rxy = np.asarray(polys["ring_xy"], np.int64)
    ro, pro = polys["ring_off"], polys["poly_ring_off"]
    on = np.zeros(len(xy), bool)
    for r in range(pro[p], pro[p + 1]):
        ring = rxy[ro[r]:ro[r + 1]]
        for a, b in zip(ring, np.roll(ring, -1, 0)):
            cross = (b[0] - a[0]) * (xy[:, 1] - a[1]) - (b[1] - a[1]) * (xy[:, 0] - a[0])
            inb = (xy[:, 0] >= min(a[0], b[0])) & (xy[:, 0] <= max(a[0], b[0])) & \
                  (xy[:, 1] >= min(a[1], b[1])) & (xy[:, 1] <= max(a[1], b[1]))
            on |= (cross == 0) & inb
    return inside | on


@pytest.mark.parametrize("seed", range(6))
def test_lattice_witnesses(seed):
    """Polygons on [0, 40]^2 scaled by 4: every lattice point of [0, 160]^2 is checked for
    membership in both closed regions.  A common lattice point forces "intersect"; polygons the
    oracle calls disjoint have no common lattice point (a necessary condition)."""
    rng = np.random.default_rng(300 + seed)
    P = _valid_polyset(rng, 7, 0, 40, scale=4)
    a, b = oracle.polygon_join(P, P)
    hit = set(zip(a.tolist(), b.tolist()))
    xs, ys = np.meshgrid(np.arange(-2, 163), np.arange(-2, 163))
    lat = np.stack([xs.ravel(), ys.ravel()], 1)
    mem = [_closed_member(lat, P, p) for p in range(7)]
    for i in range(7):
        assert (i, i) in hit
        for j in range(7):
            common = bool(np.any(mem[i] & mem[j]))
            if common:
                assert (i, j) in hit, (i, j)
            if (i, j) not in hit:
                assert not common


def _transform(polys, f):
    out = dict(polys)
    xy = np.asarray(polys["ring_xy"], np.int64)
    out["ring_xy"] = f(xy).astype(np.int32)
    return out


@pytest.mark.parametrize("seed", range(4))
def test_invariants(seed):
    rng = np.random.default_rng(400 + seed)
    A = _valid_polyset(rng, 9, 0, 60)
    B = _valid_polyset(rng, 8, 0, 60)
    a, b = oracle.polygon_join(A, B)
    ref = set(zip(a.tolist(), b.tolist()))
    b2, a2 = oracle.polygon_join(B, A)
    assert set(zip(a2.tolist(), b2.tolist())) == ref                       # symmetry
    for f in (lambda v: v + np.array([1000, -77]),                        # translation
              lambda v: v * 3,                                            # scaling
              lambda v: np.stack([-v[:, 1], v[:, 0]], 1),                 # 90-degree rotation
              lambda v: np.stack([v[:, 0], -v[:, 1]], 1),                 # reflection
              lambda v: np.stack([v[:, 1], v[:, 0]], 1)):                 # reflection in y = x
        ta, tb = oracle.polygon_join(_transform(A, f), _transform(B, f))
        assert set(zip(ta.tolist(), tb.tolist())) == ref
    # ring orientation and start vertex
    def reorder(polys):
        xy = np.asarray(polys["ring_xy"], np.int64)
        ro = polys["ring_off"]
        rings = []
        for r in range(len(ro) - 1):
            ring = xy[ro[r]:ro[r + 1]][::-1]
            rings.append(np.roll(ring, 2, 0))
        out = dict(polys)
        out["ring_xy"] = np.concatenate(rings).astype(np.int32)
        return out
    ra, rb = oracle.polygon_join(reorder(A), reorder(B))
    assert set(zip(ra.tolist(), rb.tolist())) == ref


def test_jittered_tiling_self_join_is_the_cell_adjacency():
    """A planar partition with shared wiggly borders: two cells intersect iff they share a
    border point, i.e. iff their lattice cells are at Chebyshev distance <= 1 (corners are shared
    by all four cells around them)."""
    nx, ny = 5, 4
    T = pg.jittered_tiling(nx, ny, 7, domain=1 << 16, seed=9)
    a, b = oracle.polygon_join(T, T)
    exp = {(j1 * nx + i1, j2 * nx + i2) for j1 in range(ny) for i1 in range(nx) for j2 in range(ny) for i2 in range(nx)
           if abs(i1 - i2) <= 1 and abs(j1 - j2) <= 1}
    assert set(zip(a.tolist(), b.tolist())) == exp
