"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Bar: bit-exact — counts equal, pair sets equal after sorting, selected id
sets equal.  All inputs seeded and synthetic.
"""
import numpy as np
import pytest

import gen
import oracle
from gen import configs
from gen import polygons as pg
from tests.helpers import lattice, random_polyset, sorted_pairs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def spade():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icde_doraiswamyf22_b200 as sp
    sp.load()
    return sp


def gpu_all(sp, polys, xy, s=-1, max_dim=4096, base=0, dense=False):
    import torch
    cv = sp.Canvas(polys, log2_pixel=s, max_dim=max_dim, dense=dense)
    xy_d = torch.as_tensor(np.ascontiguousarray(xy, np.int32)).cuda()
    counts = sp.join_count(cv, xy_d).cpu().numpy()
    pt, pl = sp.join_pairs(cv, xy_d, point_id_base=base)
    ids = sp.select(cv, xy_d, point_id_base=base)
    torch.cuda.synchronize()
    return cv, counts, sorted_pairs(pt.cpu().numpy(), pl.cpu().numpy()), np.sort(ids.cpu().numpy())


def check_all(sp, polys, xy, s=-1, max_dim=4096, base=0, dense=False):
    cv, counts, (pt, pl), ids = gpu_all(sp, polys, xy, s, max_dim, base, dense)
    ocounts = oracle.join_count(xy, polys)
    opt, opl = oracle.join_pairs(xy, polys, point_id_base=base)
    oids = oracle.select(xy, polys, point_id_base=base)
    np.testing.assert_array_equal(counts, ocounts)
    np.testing.assert_array_equal(pt, opt)
    np.testing.assert_array_equal(pl, opl)
    np.testing.assert_array_equal(ids, oids)
    return cv


@pytest.mark.parametrize("dense", [False, True])
@pytest.mark.parametrize("s", [-1, 0, 1, 3, 5, 8, 10])
def test_c1_all_ops_all_resolutions(spade, s, dense):
    w = configs.c1()
    xy = np.concatenate([gen.points_host(w.points, w.point_seed, 0, w.n_points), configs.c1_edge_points(w.polys)])
    check_all(spade, w.polys, xy, s=s, max_dim=w.max_dim, base=1000, dense=dense)


@pytest.mark.parametrize("seed", range(12))
def test_tiny_lattice_bruteforce(spade, seed):
    rng = np.random.default_rng(1000 + seed)
    polys = random_polyset(rng, 0, 40, int(rng.integers(1, 7)))
    xy = lattice(-2, -2, 42, 42)
    for s in (0, 1, 2, 3, 4, 6):
        check_all(spade, polys, xy, s=s, dense=bool(seed & 1))


def test_grid_tiling_closed_form(spade):
    polys = pg.grid_tiling(4, 4, 0, 0, 256, 256)
    xy = gen.points_host(gen.uniform_params(0, 0, 1024, 1024), 7, 0, 200_000)
    import torch
    for s in (-1, 0, 4, 7):
        cv = spade.Canvas(polys, log2_pixel=s)
        counts = spade.join_count(cv, torch.as_tensor(xy).cuda()).cpu().numpy()
        expect = np.bincount((xy[:, 1] >> 8) * 4 + (xy[:, 0] >> 8), minlength=16)
        np.testing.assert_array_equal(counts, expect)


def test_capacity_protocol(spade):
    import torch
    w = configs.c1()
    xy = torch.as_tensor(gen.points_host(w.points, w.point_seed, 0, w.n_points)).cuda()
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    pt, pl = spade.join_pairs(cv, xy, capacity=5)          # too small -> retry with reported size
    opt, opl = oracle.join_pairs(xy.cpu().numpy(), w.polys)
    a, b = sorted_pairs(pt.cpu().numpy(), pl.cpu().numpy())
    np.testing.assert_array_equal(a, opt)
    np.testing.assert_array_equal(b, opl)
    ids = spade.select(cv, xy, capacity=0)
    np.testing.assert_array_equal(np.sort(ids.cpu().numpy()), oracle.select(xy.cpu().numpy(), w.polys))


def test_empty_and_degenerate_inputs(spade):
    import torch
    w = configs.c1()
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    empty = torch.zeros((0, 2), dtype=torch.int32, device="cuda")
    assert spade.join_count(cv, empty).sum().item() == 0
    assert spade.select(cv, empty).numel() == 0
    # unaligned views (head / tail scalar paths) of every length 0..40
    xy = torch.as_tensor(gen.points_host(w.points, w.point_seed, 0, 64)).cuda()
    for off in range(4):
        for n in range(0, 41, 3):
            sub = xy[off:off + n]
            c = spade.join_count(cv, sub).cpu().numpy()
            np.testing.assert_array_equal(c, oracle.join_count(sub.cpu().numpy(), w.polys))
    # extreme coordinates: points far outside, at int32 limits
    far = np.array([[-2**31, -2**31], [2**31 - 1, 2**31 - 1], [-2**31, 500], [500, 2**31 - 1], [0, 0]], np.int32)
    check_all(spade, w.polys, far)
    # polygon set with no vertices at all / zero polygons
    nothing = pg.assemble([])
    cv0 = spade.Canvas(nothing)
    assert spade.join_count(cv0, xy).numel() == 0
    one_empty = {"ring_xy": np.zeros((0, 2), np.int32), "ring_off": np.zeros(1, np.int64),
                 "poly_ring_off": np.zeros(2, np.int64)}
    cv1 = spade.Canvas(one_empty)
    assert spade.join_count(cv1, xy).cpu().numpy().tolist() == [0]


def test_coord_range_error(spade):
    bad = {"ring_xy": np.array([[0, 0], [2**30, 0], [0, 5]], np.int32), "ring_off": np.array([0, 3], np.int64),
           "poly_ring_off": np.array([0, 1], np.int64)}
    with pytest.raises(spade.SpadeError) as e:
        spade.Canvas(bad)
    assert e.value.code == spade.SPADE_ERR_COORD_RANGE


def test_tiling_with_islands_exactly_one_owner(spade):
    import torch
    polys = pg.jittered_tiling(6, 5, 9, domain=1 << 20, n_islands=4, seed=5)
    xy = gen.points_host(gen.taxi_params(9, domain=1 << 20), 9, 0, 300_000)
    check_all(spade, polys, xy[:50_000])
    cv = spade.Canvas(polys)
    pt, pl = spade.join_pairs(cv, torch.as_tensor(xy).cuda())
    pt = pt.cpu().numpy()
    assert len(pt) == len(xy) and len(np.unique(pt)) == len(xy)   # every point in exactly one polygon


def test_host_streaming_count_matches_oracle(spade):
    """spade_join_count_host (host-resident points, chunked H2D overlapped with the probe)."""
    import torch
    w = configs.c1()
    xy = np.concatenate([gen.points_host(w.points, w.point_seed, 0, 300_000), configs.c1_edge_points(w.polys)])
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    got = spade.join_count_host(cv, xy)                                  # pageable numpy buffer
    np.testing.assert_array_equal(got, oracle.join_count(xy, w.polys))
    pinned = torch.from_numpy(xy).pin_memory()
    acc = np.full(cv.num_polys, 7, np.int64)                            # accumulates into counts
    spade.join_count_host(cv, pinned, acc)
    np.testing.assert_array_equal(acc - 7, got)


@pytest.mark.parametrize("chunk", [256, 4096, 1 << 25])
def test_host_streaming_select_pairs_match_oracle(spade, chunk):
    """spade_select_host / spade_join_pairs_host (NEXT(3): host-resident point streams, P:232-248,
    P:480): chunked H2D, probe and result D2H on three streams; results in chunk order."""
    import torch
    w = configs.c1()
    xy = np.concatenate([gen.points_host(w.points, w.point_seed, 0, 200_000), configs.c1_edge_points(w.polys)])
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    spade.set_option("host_chunk", chunk)
    try:
        ids = spade.select_host(cv, xy, point_id_base=77)
        pt, pl = spade.join_pairs_host(cv, torch.from_numpy(xy).pin_memory(), point_id_base=77)
        # capacity protocol: too small -> retried with the reported total
        pt2, pl2 = spade.join_pairs_host(cv, xy, point_id_base=77, capacity=5)
    finally:
        spade.set_option("host_chunk", 1 << 25)
    np.testing.assert_array_equal(np.sort(ids), oracle.select(xy, w.polys, point_id_base=77))
    opt, opl = oracle.join_pairs(xy, w.polys, point_id_base=77)
    for a, b in ((pt, pl), (pt2, pl2)):
        got = sorted_pairs(a, b)
        np.testing.assert_array_equal(got[0], opt)
        np.testing.assert_array_equal(got[1], opl)
        assert np.all(np.diff((a - 77) // min(chunk, len(xy))) >= 0)     # chunk order
    assert np.all(np.diff((ids - 77) // min(chunk, len(xy))) >= 0)


def test_host_streaming_pairs_chunk_overflow(spade):
    """Three identical squares: every chunk yields 3x its points in pairs, more than the per-chunk
    device buffer, so each chunk takes the 2-pass Map re-run."""
    sq = np.array([[0, 0], [1000, 0], [1000, 1000], [0, 1000]], np.int32)
    polys = {"ring_xy": np.concatenate([sq] * 3), "ring_off": np.array([0, 4, 8, 12], np.int64),
             "poly_ring_off": np.array([0, 1, 2, 3], np.int64)}
    rng = np.random.default_rng(3)
    xy = rng.integers(-100, 1100, size=(50_000, 2)).astype(np.int32)
    cv = spade.Canvas(polys)
    spade.set_option("host_chunk", 1000)
    try:
        pt, pl = spade.join_pairs_host(cv, xy, point_id_base=0, capacity=3 * len(xy))
    finally:
        spade.set_option("host_chunk", 1 << 25)
    opt, opl = oracle.join_pairs(xy, polys)
    got = sorted_pairs(pt, pl)
    np.testing.assert_array_equal(got[0], opt)
    np.testing.assert_array_equal(got[1], opl)
    assert len(pt) > 2 * len(xy)


def test_overlap_heavy_polygon_set(spade):
    """1,000 overlapping stars (configs.ov, NEXT(4)'s scenario): ~32 polygons per point on average,
    owner sets of dozens of polygons per pixel; all ops bit-exact against the oracle."""
    w = configs.ov()
    xy = gen.points_host(w.points, w.point_seed, 0, 30_000)
    for md in (1024, 8192):
        check_all(spade, w.polys, xy, max_dim=md, base=11)


def test_invalid_arguments_are_reported(spade):
    import ctypes
    import torch
    lib = spade.load()
    w = configs.c1()
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    xy = torch.zeros((8, 2), dtype=torch.int32, device="cuda")
    counts = torch.zeros(cv.num_polys, dtype=torch.int64, device="cuda")
    s = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    P = ctypes.c_void_p
    assert lib.spade_join_count(None, P(xy.data_ptr()), 8, P(counts.data_ptr()), s) == spade.SPADE_ERR_INVALID_ARG
    assert lib.spade_join_count(cv.handle, P(xy.data_ptr()), -1, P(counts.data_ptr()), s) == spade.SPADE_ERR_INVALID_ARG
    assert lib.spade_join_count(cv.handle, None, 8, P(counts.data_ptr()), s) == spade.SPADE_ERR_INVALID_ARG
    assert lib.spade_join_count(cv.handle, P(xy.data_ptr() + 4), 7, P(counts.data_ptr()), s) == spade.SPADE_ERR_INVALID_ARG
    assert lib.spade_join_count(cv.handle, None, 0, P(counts.data_ptr()), s) == spade.SPADE_OK   # n == 0: no-op
    n_out = ctypes.c_int64()
    assert lib.spade_select(cv.handle, P(xy.data_ptr()), 8, 0, None, 0, None, s) == spade.SPADE_ERR_INVALID_ARG
    assert lib.spade_select(cv.handle, P(xy.data_ptr()), 8, 0, None, -5, ctypes.byref(n_out), s) == spade.SPADE_ERR_INVALID_ARG
    assert b"negative" in lib.spade_last_error()
    bad = {"ring_xy": np.zeros((3, 2), np.int32), "ring_off": np.array([0, 2, 1], np.int64),
           "poly_ring_off": np.array([0, 2], np.int64)}
    with pytest.raises(spade.SpadeError) as e:
        spade.Canvas(bad)
    assert e.value.code == spade.SPADE_ERR_INVALID_ARG


def test_results_independent_of_point_id_base_and_chunking(spade):
    import torch
    w = configs.c1()
    xy = torch.as_tensor(gen.points_host(w.points, w.point_seed, 0, 50_000)).cuda()
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    full = spade.join_count(cv, xy)
    parts = torch.zeros_like(full)
    for a in range(0, 50_000, 7_919):
        spade.join_count(cv, xy[a:a + 7_919], parts)
    assert torch.equal(full, parts)
    pt, pl = spade.join_pairs(cv, xy, point_id_base=10**12)
    assert int(pt.min()) >= 10**12 and int(pt.max()) < 10**12 + 50_000


def _fan(n, R=1_000_000, overlap=False, spikes=False):
    """n triangles around the origin (adjacent ones share an edge); overlap=True adds a second
    copy of every triangle (shared edges across all polygons); spikes=True gives every triangle a
    degenerate out-and-back spur (an edge traversed twice by the same ring)."""
    th = np.linspace(0, 2 * np.pi, n + 1)
    v = np.stack([np.round(R * np.cos(th)), np.round(R * np.sin(th))], 1).astype(np.int64)
    v[-1] = v[0]
    polys = []
    for i in range(n):
        ring = [(0, 0), tuple(v[i]), tuple(v[i + 1])]
        if spikes:
            m = (v[i] + v[i + 1]) // 2
            ring = [(0, 0), tuple(v[i]), tuple(m), tuple(m * 2 - m // 3), tuple(m), tuple(v[i + 1])]
        polys.append([np.array(ring)])
    if overlap:
        polys = polys + [list(p) for p in polys]
    return pg.assemble(polys)


@pytest.mark.parametrize("n,overlap,spikes", [(40, False, False), (40, True, False), (20, True, True),
                                              (63, False, True), (100, False, False), (90, True, False)])
@pytest.mark.parametrize("s", [9, 12])
def test_many_polygons_one_pixel(spade, n, overlap, spikes, s):
    """Boundary pixels with up to 180 polygons: edges shared by 2-4 polygons are stored once
    with a polygon toggle mask (<= 64 polygons) or per polygon (> 64)."""
    polys = _fan(n, overlap=overlap, spikes=spikes)
    rng = np.random.default_rng(n + s)
    near = rng.integers(-3000, 3000, (20000, 2))
    far = rng.integers(-1_100_000, 1_100_000, (20000, 2))
    xy = np.concatenate([near, far, lattice(-40, -40, 40, 40)]).astype(np.int32)
    check_all(spade, polys, xy, s=s, max_dim=4096)


@pytest.mark.parametrize("op", ["pairs", "select"])
def test_exact_capacity_and_compaction(spade, op):
    """3M points on C1's overlapping polygons: the per-warp output chunks leave holes that are
    compacted away; with capacity exactly M the tail slots go through the overflow buffer; with
    M - 1 the call reports M; slots past the capacity are never written."""
    import ctypes
    import torch
    w = configs.c1()
    xy_h = gen.points_host(gen.uniform_params(-20, -20, 1064, 1064), 77, 0, 3_000_000)
    xy = torch.as_tensor(xy_h).cuda()
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    lib = spade.load()
    if op == "pairs":
        opt, opl = oracle.join_pairs(xy_h, w.polys, point_id_base=9)
        M = len(opt)
    else:
        oids = oracle.select(xy_h, w.polys, point_id_base=9)
        M = len(oids)
    pad = 4096
    pt = torch.full((M + pad,), -7, dtype=torch.int64, device="cuda")
    pl = torch.full((M + pad,), -7, dtype=torch.int32, device="cuda")
    n_out = ctypes.c_int64()

    def call(cap):
        if op == "pairs":
            return lib.spade_join_pairs(cv.handle, ctypes.c_void_p(xy.data_ptr()), len(xy_h), 9,
                                        ctypes.c_void_p(pt.data_ptr()), ctypes.c_void_p(pl.data_ptr()), cap,
                                        ctypes.byref(n_out), None)
        return lib.spade_select(cv.handle, ctypes.c_void_p(xy.data_ptr()), len(xy_h), 9,
                                ctypes.c_void_p(pt.data_ptr()), cap, ctypes.byref(n_out), None)

    assert call(M - 1) == spade.SPADE_ERR_CAPACITY and n_out.value == M
    pt.fill_(-7)
    pl.fill_(-7)
    assert call(M) == 0 and n_out.value == M
    torch.cuda.synchronize()
    assert bool((pt[M:] == -7).all()) and bool((pl[M:] == -7).all())
    if op == "pairs":
        a, b = sorted_pairs(pt[:M].cpu().numpy(), pl[:M].cpu().numpy())
        np.testing.assert_array_equal(a, opt)
        np.testing.assert_array_equal(b, opl)
    else:
        np.testing.assert_array_equal(np.sort(pt[:M].cpu().numpy()), oids)


def test_build_profile_and_call_stages(spade):
    """spade_canvas_build_times: one device time per build stage (CUDA events), bounded by the
    build's wall time; spade_last_call_stages: per-stage times of the last call when the
    stage_events option is on, zeros when off; results unchanged either way."""
    import time
    import torch
    w = configs.c4(1)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    torch.cuda.synchronize()
    wall_ms = 1e3 * (time.perf_counter() - t0)
    bt = cv.build_times()
    assert len(bt) == 6 and all(v >= 0 for v in bt.values())
    assert 0 < sum(bt.values()) <= wall_ms * 1.05
    xy_h = gen.points_host(w.points, w.point_seed, 0, 200_000)
    xy = torch.as_tensor(xy_h).cuda()
    spade.set_option("stage_events", 1)
    try:
        c1 = spade.join_count(cv, xy).cpu().numpy()
        st = spade.last_call_stages()
        pt, pl = spade.join_pairs(cv, xy)
        st2 = spade.last_call_stages()
    finally:
        spade.set_option("stage_events", 0)
    assert st["probe"] > 0 and st["output compaction"] < 0.05     # COUNT: no compaction (event gap only)
    assert st2["probe"] > 0 and st2["output compaction"] > 0
    c0 = spade.join_count(cv, xy).cpu().numpy()
    assert all(v == 0 for v in spade.last_call_stages().values())
    np.testing.assert_array_equal(c0, c1)
    np.testing.assert_array_equal(c0, oracle.join_count(xy_h, w.polys))
