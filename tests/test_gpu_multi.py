"""Multi-GPU readiness (-m gpu, multi-GPU is the paper's future work P:486).

* The replicated canvas: spade_canvas_checksum is deterministic (two builds of the same polygon
  arrays hash equal, on any device) and sensitive (one moved vertex changes it).
* The NCCL path: min(8, device_count) ranks each build the canvas, compare checksums, COUNT their
  contiguous shard through the CUDA path and all_reduce; every rank must hold the single-rank
  counts, PAIRS stay sharded with global ids by default and gather exactly on request, and kNN
  across the shards (default CUDA step functions) equals the single-device kNN.  On a
  one-GPU box this runs as a one-rank NCCL group (the collectives execute on the device, with
  nothing to exchange); the multi-rank exchange itself is covered there by the gloo tests.
"""
import os
import socket

import numpy as np
import pytest

import gen
import oracle
from gen import configs

pytestmark = pytest.mark.gpu


def _have_gpus(k):
    import torch
    return torch.cuda.is_available() and torch.cuda.device_count() >= k


@pytest.fixture(scope="module")
def spade():
    if not _have_gpus(1):
        pytest.skip("no CUDA device")
    import paper_conf_icde_doraiswamyf22_b200 as sp
    sp.load()
    return sp


def test_canvas_checksum_deterministic_and_sensitive(spade):
    import torch
    w = configs.c4(1)
    a = spade.canvas_checksum(spade.Canvas(w.polys, max_dim=w.max_dim))
    b = spade.canvas_checksum(spade.Canvas(w.polys, max_dim=w.max_dim))
    assert a == b
    moved = {k: v.copy() for k, v in w.polys.items()}
    moved["ring_xy"][123, 0] += 1
    assert spade.canvas_checksum(spade.Canvas(moved, max_dim=w.max_dim)) != a
    assert spade.canvas_checksum(spade.Canvas(w.polys, max_dim=w.max_dim // 2)) != a
    d = configs.dj(1, n_disks=1000)
    c1 = spade.canvas_checksum(spade.Canvas.disks(d.disks["center_xy"], d.disks["r2"], max_dim=2048))
    c2 = spade.canvas_checksum(spade.Canvas.disks(d.disks["center_xy"], d.disks["r2"], max_dim=2048))
    assert c1 == c2
    if _have_gpus(2):                                   # another device builds the same canvas
        with torch.cuda.device(1):
            assert spade.canvas_checksum(spade.Canvas(w.polys, max_dim=w.max_dim)) == a


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


N = 3_000_000


def _nccl_worker(rank, world, port, out):
    import torch
    import torch.distributed as dist
    import paper_conf_icde_doraiswamyf22_b200 as sp
    from paper_conf_icde_doraiswamyf22_b200 import distributed as sd
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    try:
        w = configs.c4(N)
        cv = sp.Canvas(w.polys, max_dim=w.max_dim)
        agree = sd.canvas_checksums_agree(cv)
        a, b = sd.shard_range(N, rank, world)
        xy = gen.points_device(w.points, w.point_seed, a, b - a)
        counts = sd.join_count_distributed(cv, xy)
        pt, pl = sd.join_pairs_distributed(cv, xy, a)             # sharded (default)
        sharded_ok = bool(pt.numel() == b - a and int(pt.min()) >= a and int(pt.max()) < b)
        g = sd.join_pairs_distributed(cv, xy, a, gather=True, dst=0)
        # kNN across the shards with the default (CUDA) step functions
        ki, kd = sd.knn_distributed(xy, (8_400_000, 8_300_000), 50, a)
        res = {"agree": agree, "counts": counts.cpu().numpy().tolist(), "sharded_ok": sharded_ok,
               "knn": (ki.cpu().numpy(), kd.cpu().numpy())}
        if rank == 0:
            res["gathered"] = (g[0].cpu().numpy(), g[1].cpu().numpy())
        out[rank] = res
    finally:
        dist.destroy_process_group()


def test_nccl_count_pairs_and_checksums(spade):
    import torch
    import torch.multiprocessing as mp
    world = min(8, torch.cuda.device_count())
    w = configs.c4(N)
    cv = spade.Canvas(w.polys, max_dim=w.max_dim)
    ref = spade.join_count(cv, gen.points_device(w.points, w.point_seed, 0, N)).cpu().numpy()
    ctx = mp.get_context("spawn")
    mgr = ctx.Manager()
    out = mgr.dict()
    mp.start_processes(_nccl_worker, args=(world, _free_port(), out), nprocs=world, join=True, start_method="spawn")
    for r in range(world):
        assert out[r]["agree"]
        assert out[r]["sharded_ok"]
        np.testing.assert_array_equal(np.array(out[r]["counts"]), ref)
    xy_all = gen.points_device(w.points, w.point_seed, 0, N)
    ri, rd = spade.knn(xy_all, (8_400_000, 8_300_000), 50)
    for r in range(world):
        np.testing.assert_array_equal(out[r]["knn"][0], ri.cpu().numpy())
        np.testing.assert_array_equal(out[r]["knn"][1], rd.cpu().numpy())
    gpt, gpl = out[0]["gathered"]
    assert len(gpt) == N and len(np.unique(gpt)) == N
    np.testing.assert_array_equal(np.bincount(gpl, minlength=len(ref)), ref)
    idx = np.random.default_rng(3).integers(0, N, 2000)
    lab = np.full(N, -1, np.int64)
    lab[gpt] = gpl
    xs = gen.points_at(w.points, w.point_seed, idx)
    opt, opl = oracle.join_pairs(xs, w.polys)
    exp = np.full(len(idx), -1, np.int64)
    exp[opt] = opl
    np.testing.assert_array_equal(lab[idx], exp)
