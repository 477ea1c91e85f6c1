"""GPU parity of every probe path: the COUNT / SELECT / PAIRS results must equal the oracle's
whichever path the launcher takes (in-loop warp queues, the deferral kernel, the cooperative
deferred COUNT kernel with 4 / 8 / 16 lanes per point, global counters with and without the
shared-memory count cache).  The paths are forced with spade_set_option (include/spade.h), so
small inputs cover the branches that large configurations (C5's 40k polygons, dj2's 100K disks)
take by default.  Bit-exact, like every parity test.
"""
import numpy as np
import pytest

import gen
import oracle
from gen import configs
from gen import polygons as pg
from tests.helpers import lattice, random_polyset, sorted_pairs

pytestmark = pytest.mark.gpu

DEFAULTS = {"defer": 0, "count_global": 0, "global_queue": 0, "cache_slots": 4096, "coop": 0, "pipe": -1,
            "defer_xy": 0, "multi_agg": 1, "k_agg": -1, "tma": 0, "fine16": 1, "pipe_notile": 0,
            "hist_copies_max": 16, "idx_queue": -1}

COUNT_PATHS = [
    {},
    {"defer": 1},
    {"defer": 1, "coop": -1},
    {"defer": 1, "coop": 4},
    {"defer": 1, "coop": 8},
    {"defer": 1, "coop": 16},
    {"count_global": 1},
    {"count_global": 1, "cache_slots": 0, "coop": 0},
    {"count_global": 1, "cache_slots": 1024, "coop": 16},
    {"count_global": 1, "global_queue": 1},
    {"count_global": 1, "global_queue": 1, "cache_slots": 0},
    {"pipe": 1},
    {"pipe": 1, "count_global": 1},
    {"pipe": 1, "count_global": 1, "cache_slots": 0},
    {"pipe": 1, "defer_xy": 1},
    {"pipe": 1, "count_global": 1, "defer_xy": 1, "coop": 8},
    {"pipe": 0, "defer": 1},
    {"multi_agg": 0},
    {"multi_agg": 0, "count_global": 1},
    {"multi_agg": 0, "pipe": 1},
    {"k_agg": 1},
    {"k_agg": 1, "defer": 1},
    {"k_agg": 1, "count_global": 1},
    {"k_agg": 1, "count_global": 1, "defer": 1},
    {"k_agg": 1, "pipe": 1},
    {"k_agg": 1, "multi_agg": 0, "pipe": 1, "count_global": 1},
    {"tma": 1},
    {"pipe": 1, "pipe_notile": 1},
    {"tma": 1, "k_agg": 1},
    {"fine16": 0, "pipe": 1},
    {"idx_queue": 1},
    {"idx_queue": -1, "hist_copies_max": 32},
    {"idx_queue": 1, "k_agg": 1},
    {"hist_copies_max": 8, "idx_queue": 0},
    {"hist_copies_max": 1, "idx_queue": 1},
    {"hist_copies_max": 16, "multi_agg": 0},
    {"hist_copies_max": 1},                         # an odd-sized histogram before the 8-B point queue
    {"hist_copies_max": 1, "k_agg": 1},
]


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


def _polygon_cases():
    w = configs.c1()
    c1_xy = np.concatenate([gen.points_host(w.points, w.point_seed, 0, w.n_points), configs.c1_edge_points(w.polys)])
    cases = [("c1_s0", w.polys, c1_xy, 0), ("c1_s3", w.polys, c1_xy, 3), ("c1_s8", w.polys, c1_xy, 8)]
    for seed in range(3):
        rng = np.random.default_rng(500 + seed)
        cases.append((f"rand{seed}", random_polyset(rng, 0, 40, int(rng.integers(2, 7))), lattice(-2, -2, 42, 42), seed))
    til = pg.jittered_tiling(6, 5, 12, domain=1 << 20, n_islands=3, seed=77)
    til_xy = gen.points_host(gen.uniform_params(-1000, -1000, (1 << 20) + 2000, (1 << 20) + 2000), 78, 0, 200_000)
    cases.append(("tiling_s9", til, til_xy, 9))      # long edges: absolute (int4) primitives
    cases.append(("tiling_s12", til, til_xy, 12))
    return cases


POLY_CASES = _polygon_cases()


@pytest.mark.parametrize("opts", COUNT_PATHS, ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()) or "default")
@pytest.mark.parametrize("case", POLY_CASES, ids=lambda c: c[0])
def test_count_paths_polygons(spade, case, opts):
    import torch
    name, polys, xy, s = case
    _set(spade, opts)
    try:
        cv = spade.Canvas(polys, log2_pixel=s)
        counts = spade.join_count(cv, torch.as_tensor(np.ascontiguousarray(xy, np.int32)).cuda()).cpu().numpy()
    finally:
        _set(spade, {})
    np.testing.assert_array_equal(counts, oracle.join_count(xy, polys))


def _fan(n):
    v = np.stack([np.round(1e6 * np.cos(np.linspace(0, 2 * np.pi, n + 1))),
                  np.round(1e6 * np.sin(np.linspace(0, 2 * np.pi, n + 1)))], 1).astype(np.int64)
    return pg.assemble([[np.array([(0, 0), tuple(v[i]), tuple(v[i + 1])])] for i in range(n)] * 2)


@pytest.mark.parametrize("opts", [{"defer": 1}, {"count_global": 1}, {"count_global": 1, "coop": 0}],
                         ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
def test_count_paths_more_than_64_polygons_per_pixel(spade, opts):
    """Records with > 64 polygons are evaluated serially by the cooperative kernel's first lane."""
    import torch
    polys = _fan(90)
    rng = np.random.default_rng(3)
    xy = np.concatenate([rng.integers(-3000, 3000, (20000, 2)), lattice(-40, -40, 40, 40)]).astype(np.int32)
    _set(spade, opts)
    try:
        cv = spade.Canvas(polys, log2_pixel=9)
        counts = spade.join_count(cv, torch.as_tensor(xy).cuda()).cpu().numpy()
    finally:
        _set(spade, {})
    np.testing.assert_array_equal(counts, oracle.join_count(xy, polys))


@pytest.mark.parametrize("opts", COUNT_PATHS[1:], ids=lambda o: ",".join(f"{k}={v}" for k, v in o.items()))
def test_count_paths_disks(spade, opts):
    import torch
    rng = np.random.default_rng(11)
    cxy = rng.integers(0, 60, (40, 2))
    disks = {"center_xy": np.ascontiguousarray(cxy, np.int32), "r2": rng.integers(0, 400, 40).astype(np.int64)}
    xy = lattice(-25, -25, 85, 85)
    _set(spade, opts)
    try:
        for s in (0, 2, 4):
            cv = spade.Canvas.disks(disks["center_xy"], disks["r2"], log2_pixel=s)
            counts = spade.join_count(cv, torch.as_tensor(xy).cuda()).cpu().numpy()
            np.testing.assert_array_equal(counts, oracle.disk_join_count(xy, disks))
    finally:
        _set(spade, {})


@pytest.mark.parametrize("case", POLY_CASES, ids=lambda c: c[0])
def test_select_pairs_deferred_path(spade, case):
    """SELECT / PAIRS through the deferral kernel (forced) equal the oracle."""
    import torch
    name, polys, xy, s = case
    _set(spade, {"defer": 1})
    try:
        cv = spade.Canvas(polys, log2_pixel=s)
        xy_d = torch.as_tensor(np.ascontiguousarray(xy, np.int32)).cuda()
        pt, pl = spade.join_pairs(cv, xy_d, point_id_base=7)
        ids = spade.select(cv, xy_d, point_id_base=7)
        torch.cuda.synchronize()
    finally:
        _set(spade, {})
    opt, opl = oracle.join_pairs(xy, polys, point_id_base=7)
    gpt, gpl = sorted_pairs(pt.cpu().numpy(), pl.cpu().numpy())
    np.testing.assert_array_equal(gpt, opt)
    np.testing.assert_array_equal(gpl, opl)
    np.testing.assert_array_equal(np.sort(ids.cpu().numpy()), oracle.select(xy, polys, point_id_base=7))


def test_set_option_rejects_bad_values(spade):
    with pytest.raises(spade.SpadeError):
        spade.set_option("coop", 3)
    with pytest.raises(spade.SpadeError):
        spade.set_option("no_such_option", 1)
    with pytest.raises(spade.SpadeError):
        spade.set_option("cache_slots", 1000)
