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
