"""GPU parity of the Polygon x Polygon join (spade_join_polygons; reading C15:
closed regions intersect) against the brute-force oracle (oracle/polygon_join_oracle.c), pair
sets identical (both sorted by (a, b)).  Cases: the hand cases of the oracle pins, random valid
polygon sets (stars, holes, two-component polygons) at several grid resolutions, touching grids
and wiggly tilings (shared borders: every adjacent pair by contact), overlapping stars, the C4
census-like tiling against the C3 neighbourhood-like tiling (2,200 x 260 polygons), and the
rotation invariance of the closed predicate.
"""
import json
import os

import numpy as np
import pytest

import oracle
from gen import configs
from gen import polygons as pg
from tests.helpers import valid_polyset

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def spade():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icde_doraiswamyf22_b200 as sp
    sp.load()
    return sp


def _gpu(sp, A, B, **kw):
    a, b = sp.join_polygons(A, B, **kw)
    return a.cpu().numpy().astype(np.int64), b.cpu().numpy().astype(np.int64)


def _check(sp, A, B, **kw):
    ga, gb = _gpu(sp, A, B, **kw)
    oa, ob = oracle.polygon_join(A, B)
    np.testing.assert_array_equal(ga, oa)
    np.testing.assert_array_equal(gb, ob)
    return len(oa)


def test_hand_cases(spade):
    cases = json.load(open(os.path.join(ROOT, "tests", "golden", "polygon_join_cases.json")))["cases"]
    for c in cases:
        A = pg.assemble([[np.array(r, np.int64) for r in c["A"]]])
        B = pg.assemble([[np.array(r, np.int64) for r in c["B"]]])
        for s in (-1, 0, 2, 3):
            a, b = _gpu(spade, A, B, log2_pixel=s)
            assert (len(a) == 1) == c["expect"], (c["name"], s)


@pytest.mark.parametrize("seed", range(8))
def test_random_valid_sets_all_resolutions(spade, seed):
    rng = np.random.default_rng(900 + seed)
    A = valid_polyset(rng, 14, 0, 60, scale=16)
    B = valid_polyset(rng, 11, 0, 60, scale=16)
    for s in (-1, 0, 3, 5, 7, 9):
        _check(spade, A, B, log2_pixel=s)


def test_touching_grids_and_tilings(spade):
    G = pg.grid_tiling(6, 5, 0, 0, 1000, 700)
    H = pg.grid_tiling(6, 5, 500, 350, 1000, 700)
    assert _check(spade, G, G) == sum(1 for j in range(5) for i in range(6) for j2 in range(5) for i2 in range(6)
                                      if abs(i - i2) <= 1 and abs(j - j2) <= 1)
    _check(spade, G, H, log2_pixel=6)
    T = pg.jittered_tiling(7, 6, 9, domain=1 << 20, n_islands=3, seed=12)
    U = pg.jittered_tiling(5, 4, 13, domain=1 << 20, seed=13)
    for s in (-1, 8, 12):
        _check(spade, T, T, log2_pixel=s)
        _check(spade, T, U, log2_pixel=s)


def test_overlapping_stars(spade):
    w = configs.ov(1, n_polys=150)
    rng = np.random.default_rng(5)
    B = valid_polyset(rng, 60, 0, 1 << 10, scale=1 << 14)
    _check(spade, w.polys, w.polys)
    _check(spade, w.polys, B, max_dim=2048)


def test_rotation_invariance(spade):
    rng = np.random.default_rng(77)
    A = valid_polyset(rng, 20, 0, 80, scale=8)
    B = valid_polyset(rng, 20, 0, 80, scale=8)
    ref = _gpu(spade, A, B)

    def rot(P):
        out = dict(P)
        xy = np.asarray(P["ring_xy"], np.int64)
        out["ring_xy"] = np.stack([-xy[:, 1], xy[:, 0]], 1).astype(np.int32)
        return out
    got = _gpu(spade, rot(A), rot(B))
    np.testing.assert_array_equal(got[0], ref[0])
    np.testing.assert_array_equal(got[1], ref[1])


def test_capacity_protocol(spade):
    import ctypes
    import torch
    G = pg.grid_tiling(4, 4, 0, 0, 100, 100)
    a, b = spade.join_polygons(G, G, capacity=3)          # too small -> retried with the reported size
    oa, ob = oracle.polygon_join(G, G)
    np.testing.assert_array_equal(a.cpu().numpy(), oa)
    lib = spade.load()
    d = [torch.as_tensor(np.ascontiguousarray(G[k])).cuda() for k in ("ring_xy", "ring_off", "poly_ring_off")]
    out = torch.full((5,), -1, dtype=torch.int32, device="cuda")
    n_out = ctypes.c_int64()
    P = ctypes.c_void_p
    rc = lib.spade_join_polygons(P(d[0].data_ptr()), P(d[1].data_ptr()), P(d[2].data_ptr()), 16,
                                 P(d[0].data_ptr()), P(d[1].data_ptr()), P(d[2].data_ptr()), 16, None,
                                 P(out.data_ptr()), P(out.data_ptr()), 0, ctypes.byref(n_out), None)
    assert rc == spade.SPADE_ERR_CAPACITY and n_out.value == len(oa)
    assert bool((out == -1).all())


@pytest.mark.slow
def test_census_x_neighbourhoods_full_size(spade):
    """C4's 2,200 census-like polygons (holes, islands) against C3's 260 neighbourhood-like
    polygons, at the canvas resolution bench.py uses for the pp workload."""
    A = configs.c4(1).polys
    B = configs.c3(1).polys
    n = _check(spade, A, B, max_dim=8192)
    assert n > 2200
