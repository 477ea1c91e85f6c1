"""Multi-rank combine logic on CPU (gloo, world_size 2), the oracle standing in for the GPU.

Checks: shard ranges partition [0, N); per-rank COUNT + all_reduce equals the single-process
count; gathered pairs equal the single-process pairs; shard count does not change results.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle
from gen import polygons as pg
from paper_conf_icde_doraiswamyf22_b200 import distributed as sd

N = 20_000


def _polys():
    return pg.jittered_tiling(4, 3, 10, domain=1 << 20, n_islands=2, seed=8)


def _points(start, n):
    return gen.points_host(gen.taxi_params(12, domain=1 << 20), 12, start, n)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        polys = _polys()
        start, stop = sd.shard_range(N, rank, world)
        xy = _points(start, stop - start)
        cnt = sd.join_count_distributed(polys, xy, count_fn=lambda p, x: torch.from_numpy(oracle.join_count(x, p, 2)))
        pt, pl = oracle.join_pairs(xy, polys, point_id_base=start, nthreads=2)
        g = sd.gather_pairs(torch.from_numpy(pt), torch.from_numpy(pl.astype(np.int64)), dst=0)
        out[rank] = (cnt.numpy().tolist(), None if g is None else (g[0].numpy().tolist(), g[1].numpy().tolist()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_count_and_pairs_equal_single_process(world):
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), out), nprocs=world, join=True)
    polys = _polys()
    xy = _points(0, N)
    ref_counts = oracle.join_count(xy, polys).tolist()
    rpt, rpl = oracle.join_pairs(xy, polys)
    for r in range(world):
        assert out[r][0] == ref_counts                      # every rank holds the global counts
    gpt, gpl = out[0][1]
    o = np.lexsort((np.array(gpl), np.array(gpt)))
    assert np.array(gpt)[o].tolist() == rpt.tolist()
    assert np.array(gpl)[o].tolist() == rpl.tolist()
    assert sum(ref_counts) == N                             # tiling: every point exactly once


def test_shard_ranges_partition():
    for n in (0, 1, 7, 1000, 10**9 + 7):
        for w in (1, 2, 3, 8):
            rs = [sd.shard_range(n, r, w) for r in range(w)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(w - 1))
            assert max(b - a for a, b in rs) - min(b - a for a, b in rs) <= 1


# ---- kNN over sharded points: histogram all_reduce, shared radius, candidate all_gather ----

def _bucket(d2):
    d2 = np.asarray(d2, np.int64)
    out = d2.copy()
    big = d2 >= 4
    e = np.floor(np.log2(np.maximum(d2, 1))).astype(np.int64)
    # exact floor(log2) for int64 (float rounding near powers of two)
    e = np.where((1 << np.clip(e, 0, 62)) > d2, e - 1, e)
    e = np.where((1 << np.clip(e + 1, 0, 62)) <= d2, e + 1, e)
    out[big] = 4 + 4 * (e[big] - 2) + ((d2[big] >> (e[big] - 2)) & 3)
    return out


def _knn_worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        start, stop = sd.shard_range(N, rank, world)
        xy = _points(start, stop - start)
        q = (400_000, 500_000)

        def hist_fn(x, q_):
            d2 = ((x.astype(np.int64) - np.array(q_)) ** 2).sum(1)
            return torch.from_numpy(np.bincount(_bucket(d2), minlength=249).astype(np.int64))

        def select_fn(x, q_, r2, base):
            d2 = ((x.astype(np.int64) - np.array(q_)) ** 2).sum(1)
            m = d2 <= r2
            return torch.from_numpy(np.nonzero(m)[0].astype(np.int64) + base), torch.from_numpy(d2[m])

        def topk_fn(ids, d2, k):
            o = np.lexsort((ids.numpy(), d2.numpy()))[:k]
            return ids[o], d2[o]

        from paper_conf_icde_doraiswamyf22_b200 import knn_radius
        res = {}
        for k in (1, 17, 500):
            ids, d2 = sd.knn_distributed(xy, q, k, start, hist_fn, knn_radius, select_fn, topk_fn)
            res[k] = (ids.numpy().tolist(), d2.numpy().tolist())
        out[rank] = res
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_knn_equals_oracle(world):
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_knn_worker, args=(world, _free_port(), out), nprocs=world, join=True)
    xy = _points(0, N)
    for k in (1, 17, 500):
        oi, od = oracle.knn(xy, (400_000, 500_000), k)
        for r in range(world):
            assert out[r][k][0] == oi.tolist()
            assert out[r][k][1] == od.tolist()


# ---- sharded outputs by default, exact-size gather on request, replicated-canvas checksums ----

def _shard_worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        polys = _polys()
        start, stop = sd.shard_range(N, rank, world)
        xy = _points(start, stop - start)

        def pairs_fn(p, x, base):
            pt, pl = oracle.join_pairs(x, p, point_id_base=base, nthreads=2)
            return torch.from_numpy(pt), torch.from_numpy(pl.astype(np.int64))

        def select_fn(p, x, base):
            return torch.from_numpy(oracle.select(x, p, point_id_base=base, nthreads=2))

        local = sd.join_pairs_distributed(polys, xy, start, pairs_fn=pairs_fn)
        gathered = sd.join_pairs_distributed(polys, xy, start, pairs_fn=pairs_fn, gather=True, dst=world - 1)
        ids = sd.select_distributed(polys, xy, start, select_fn=select_fn, gather=True, dst=0)
        agree = sd.canvas_checksums_agree(polys, checksum_fn=lambda p: 0xDEADBEEFCAFEF00D)
        differ = sd.canvas_checksums_agree(polys, checksum_fn=lambda p: 12345 + (rank == 1))
        empty = sd.gather_variable(torch.zeros(0, dtype=torch.int64) if rank != 0 else torch.arange(5), dst=1)
        out[rank] = {"local": (local[0].numpy().tolist(), local[1].numpy().tolist()),
                     "gathered": None if gathered is None else (gathered[0].numpy().tolist(), gathered[1].numpy().tolist()),
                     "ids": None if ids is None else ids.numpy().tolist(), "agree": agree, "differ": differ,
                     "empty": None if empty is None else empty.numpy().tolist(), "range": (start, stop)}
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_outputs_gather_on_request_and_checksums(world):
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_shard_worker, args=(world, _free_port(), out), nprocs=world, join=True)
    polys = _polys()
    xy = _points(0, N)
    rpt, rpl = oracle.join_pairs(xy, polys)
    for r in range(world):
        a, b = out[r]["range"]
        lpt = np.array(out[r]["local"][0])
        assert len(lpt) == 0 or (lpt.min() >= a and lpt.max() < b)      # sharded: own ids only
        m = (rpt >= a) & (rpt < b)
        o = np.lexsort((np.array(out[r]["local"][1]), lpt))
        assert lpt[o].tolist() == rpt[m].tolist()
        assert out[r]["agree"] is True
        assert out[r]["differ"] is False
        assert (out[r]["gathered"] is None) == (r != world - 1)
        assert (out[r]["ids"] is None) == (r != 0)
    gpt, gpl = out[world - 1]["gathered"]
    o = np.lexsort((np.array(gpl), np.array(gpt)))
    assert np.array(gpt)[o].tolist() == rpt.tolist()
    assert np.array(gpl)[o].tolist() == rpl.tolist()
    assert sorted(out[0]["ids"]) == oracle.select(xy, polys).tolist()
    assert out[1]["empty"] == [0, 1, 2, 3, 4]
