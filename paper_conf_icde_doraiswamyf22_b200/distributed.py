"""Multi-GPU combine for the join (the paper has no multi-GPU design).

Points shard by contiguous global index ranges; every rank builds the same canvas (replicated,
identical polygon arrays); per-rank results combine with one collective:
  * COUNT: all_reduce(SUM) of int64[P]                      (NCCL over NVLink on B200)
  * PAIRS / SELECT: sizes all_gather + padded gather to one rank, or left sharded with
    global ids (point_id_base = first global index of the shard).
The per-rank compute function is injectable so the host-side logic runs under gloo on CPU in
the tests (with the oracle standing in for the GPU); on GPUs it is the CUDA path.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """[start, stop) of the contiguous global-index shard of `rank` (balanced to +-1)."""
    return (n_total * rank) // world, (n_total * (rank + 1)) // world


def allreduce_counts(counts: torch.Tensor, group=None) -> torch.Tensor:
    """Sum per-polygon int64 counts over all ranks, in place (the only exchange of COUNT)."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    return counts


def join_count_distributed(canvas, xy_shard, count_fn=None, group=None) -> torch.Tensor:
    """COUNT of this rank's shard, then all_reduce: every rank ends with the global counts."""
    if count_fn is None:
        from . import join_count as count_fn
    counts = count_fn(canvas, xy_shard)
    return allreduce_counts(counts, group)


def gather_variable(t: torch.Tensor, dst: int = 0, group=None):
    """Gather 1-D tensors of different lengths to rank `dst` (all_gather of sizes, pad, gather).
    Returns the concatenation (rank order) on dst, None elsewhere."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    n = torch.tensor([t.numel()], dtype=torch.int64, device=t.device)
    sizes = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(sizes, n, group=group)
    sizes = [int(s.item()) for s in sizes]
    m = max(sizes) if sizes else 0
    padded = torch.zeros(max(m, 1), dtype=t.dtype, device=t.device)
    padded[: t.numel()] = t
    bufs = [torch.zeros_like(padded) for _ in range(world)] if rank == dst else None
    dist.gather(padded, bufs, dst=dst, group=group)
    if rank != dst:
        return None
    return torch.cat([b[:s] for b, s in zip(bufs, sizes)])


def gather_pairs(point_ids: torch.Tensor, poly_ids: torch.Tensor, dst: int = 0, group=None):
    """Per-rank (global point id, polygon id) pairs -> all pairs on rank dst (order: by rank)."""
    a = gather_variable(point_ids, dst, group)
    b = gather_variable(poly_ids, dst, group)
    return (a, b) if a is not None else None


def all_gather_variable(t: torch.Tensor, group=None) -> torch.Tensor:
    """Concatenation (rank order) of 1-D tensors of different lengths, on every rank."""
    world = dist.get_world_size(group)
    n = torch.tensor([t.numel()], dtype=torch.int64, device=t.device)
    sizes = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(sizes, n, group=group)
    sizes = [int(s.item()) for s in sizes]
    m = max(sizes) if sizes else 0
    padded = torch.zeros(max(m, 1), dtype=t.dtype, device=t.device)
    padded[: t.numel()] = t
    bufs = [torch.zeros_like(padded) for _ in range(world)]
    dist.all_gather(bufs, padded, group=group)
    return torch.cat([b[:s] for b, s in zip(bufs, sizes)])


def knn_distributed(xy_shard, q, k: int, point_id_base: int, hist_fn=None, radius_fn=None, select_fn=None,
                    topk_fn=None, group=None):
    """kNN selection over points sharded across ranks (multi-GPU is the
    paper's future work).  The three steps with one exchange each:
      1. circle aggregation per shard, then all_reduce(SUM) of the int64 circle histogram;
      2. every rank picks the same circle (smallest with COUNT >= k) and selects its candidates;
      3. candidates all_gather'ed, then sorted by (dist2, id): every rank holds the same top k.
    The per-step functions default to the CUDA path (knn_histogram / knn_radius / knn_select /
    knn_topk) and are injectable so the combine logic runs under gloo on CPU in the tests."""
    if hist_fn is None:
        from . import knn_histogram as hist_fn
    if radius_fn is None:
        from . import knn_radius as radius_fn
    if select_fn is None:
        from . import knn_select
        select_fn = lambda xy, q_, r2, base: knn_select(xy, q_, r2, point_id_base=base)  # noqa: E731
    if topk_fn is None:
        from . import knn_topk as topk_fn
    hist = hist_fn(xy_shard, q)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(hist, op=dist.ReduceOp.SUM, group=group)
    h = hist.cpu().numpy()
    if h[-1] > 0:
        raise ValueError(f"knn: {int(h[-1])} points outside [-2^30, 2^30)")
    r2, _ = radius_fn(h, k)
    ids, d2 = select_fn(xy_shard, q, r2, point_id_base)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        ids = all_gather_variable(ids, group)
        d2 = all_gather_variable(d2, group)
    return topk_fn(ids, d2, k)
