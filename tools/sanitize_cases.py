"""Small end-to-end cases for compute-sanitizer (memcheck / racecheck / synccheck / initcheck).

Runs C1 and reduced C2 / C4 / ov / disk / kNN inputs through every COUNT probe path of
tests/test_gpu_paths.py (COUNT_PATHS), SELECT / PAIRS through the in-loop queues and the
deferral kernel (with and without a forced launch split), the host-streaming calls and the kNN
steps, and checks every result against the oracle (so a sanitizer run is also a parity run).

    compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_cases.py [--quick]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icde_doraiswamyf22_b200 as sp  # noqa: E402
from gen import configs  # noqa: E402
from tests.helpers import sorted_pairs  # noqa: E402
from tests.test_gpu_paths import COUNT_PATHS, DEFAULTS  # noqa: E402

DEF = {**DEFAULTS, "max_launch_points": (1 << 31) - 64}


def setopts(o):
    for k, v in DEF.items():
        sp.set_option(k, o.get(k, v))


def cases(quick):
    w1 = configs.c1()
    c1_xy = np.concatenate([gen.points_host(w1.points, w1.point_seed, 0, 20_000), configs.c1_edge_points(w1.polys)])
    out = [("c1", w1.polys, c1_xy, w1.max_dim)]
    if not quick:
        w2 = configs.c2(60_000)
        out.append(("c2", w2.polys, gen.points_host(w2.points, w2.point_seed, 0, 60_000), 1024))
        w4 = configs.c4(60_000)
        out.append(("c4", w4.polys, gen.points_host(w4.points, w4.point_seed, 0, 60_000), 2048))
        wo = configs.ov(20_000, n_polys=120)
        out.append(("ov", wo.polys, gen.points_host(wo.points, wo.point_seed, 0, 20_000), 1024))
    return out


def main():
    quick = "--quick" in sys.argv
    sp.load()
    n_checks = 0
    for name, polys, xy, md in cases(quick):
        xy_d = torch.as_tensor(np.ascontiguousarray(xy, np.int32)).cuda()
        oc = oracle.join_count(xy, polys)
        opt, opl = oracle.join_pairs(xy, polys, point_id_base=11)
        osel = oracle.select(xy, polys, point_id_base=11)
        for opts in COUNT_PATHS + [{"max_launch_points": 4099}, {"max_launch_points": 4099, "defer": 1, "k_agg": 1}]:
            setopts(opts)
            cv = sp.Canvas(polys, max_dim=md)
            c = sp.join_count(cv, xy_d).cpu().numpy()
            assert np.array_equal(c, oc), (name, opts)
            n_checks += 1
            del cv
        for opts in ({}, {"defer": 1}, {"defer": 1, "max_launch_points": 4099}, {"max_launch_points": 4099}):
            setopts(opts)
            cv = sp.Canvas(polys, max_dim=md)
            pt, pl = sp.join_pairs(cv, xy_d, point_id_base=11, capacity=len(opt) + 1)
            a, b = sorted_pairs(pt.cpu().numpy(), pl.cpu().numpy())
            assert np.array_equal(a, opt) and np.array_equal(b, opl), (name, opts)
            ids = sp.select(cv, xy_d, point_id_base=11)
            assert np.array_equal(np.sort(ids.cpu().numpy()), osel), (name, opts)
            n_checks += 2
        setopts({"host_chunk": 4096})
        cv = sp.Canvas(polys, max_dim=md)
        assert np.array_equal(sp.join_count_host(cv, xy), oc)
        hp, hl = sp.join_pairs_host(cv, xy, point_id_base=11)
        a, b = sorted_pairs(hp, hl)
        assert np.array_equal(a, opt) and np.array_equal(b, opl)
        n_checks += 2
        setopts({})
        sp.set_option("host_chunk", 1 << 25)
        print(f"{name}: ok", flush=True)
    # disks + kNN
    rng = np.random.default_rng(11)
    disks = {"center_xy": rng.integers(0, 60, (40, 2)).astype(np.int32), "r2": rng.integers(0, 400, 40).astype(np.int64)}
    xy = np.stack(np.meshgrid(np.arange(-25, 86), np.arange(-25, 86)), -1).reshape(-1, 2).astype(np.int32)
    for opts in ({}, {"defer": 1}, {"count_global": 1}, {"pipe": 1}):
        setopts(opts)
        cv = sp.Canvas.disks(disks["center_xy"], disks["r2"], log2_pixel=2)
        assert np.array_equal(sp.join_count(cv, torch.as_tensor(xy).cuda()).cpu().numpy(), oracle.disk_join_count(xy, disks))
        n_checks += 1
    setopts({})
    xk = gen.points_host(gen.taxi_params(5), 5, 0, 50_000)
    ids, d2 = sp.knn(torch.as_tensor(xk).cuda(), (1 << 23, 1 << 23), 37)
    oi, od = oracle.knn(xk, (1 << 23, 1 << 23), 37)
    assert np.array_equal(ids.cpu().numpy(), oi) and np.array_equal(d2.cpu().numpy(), od)
    n_checks += 1
    cv = sp.Canvas(configs.c1().polys, max_dim=1024)
    sp.canvas_checksum(cv)
    # polygon x polygon join
    from tests.helpers import valid_polyset
    rng = np.random.default_rng(3)
    A, B = valid_polyset(rng, 12, 0, 60, scale=16), valid_polyset(rng, 9, 0, 60, scale=16)
    for s_ in (-1, 4):
        a, b = sp.join_polygons(A, B, log2_pixel=s_)
        oa, ob = oracle.polygon_join(A, B)
        assert np.array_equal(a.cpu().numpy(), oa) and np.array_equal(b.cpu().numpy(), ob)
        n_checks += 1
    # the layer index (one canvas and one pass per layer) over an overlapping valid set
    from tests.helpers import lattice
    xl = lattice(-2, -2, 62, 62) * 16
    lc = sp.LayeredCanvas(A, max_dim=256)
    got = sp.join_count_layered(lc, torch.as_tensor(xl.astype(np.int32)).cuda()).cpu().numpy()
    assert np.array_equal(got, oracle.join_count(xl.astype(np.int32), A))
    n_checks += 1
    torch.cuda.synchronize()
    print(f"sanitize cases: {n_checks} checks ok, {sp.launch_count()} kernel launches", flush=True)


if __name__ == "__main__":
    main()
