"""Multi-GPU combine for the join (the paper has no multi-GPU design).

Points shard by contiguous global index ranges; every rank builds the same canvas (replicated,
identical polygon arrays; `canvas_checksums_agree` verifies it); per-rank results combine with
one collective:
  * COUNT: all_reduce(SUM) of int64[P]                      (NCCL over NVLink on B200)
  * PAIRS / SELECT: left SHARDED by default — each rank keeps its own results with global point
    ids (point_id_base = first global index of its shard); `gather=True` collects them on one
    rank (sizes all_gather, then exact-size point-to-point transfers: no padding, no buffer
    larger than the result on the destination).
The per-rank compute function is injectable so the host-side logic runs under gloo on CPU in
the tests (with the oracle standing in for the GPU); on GPUs it is the CUDA path.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def _multi(group=None) -> bool:
    return dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1


def shard_range(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """[start, stop) of the contiguous global-index shard of `rank` (balanced to +-1)."""
    return (n_total * rank) // world, (n_total * (rank + 1)) // world


def allreduce_counts(counts: torch.Tensor, group=None) -> torch.Tensor:
    """Sum per-polygon int64 counts over all ranks, in place (the only exchange of COUNT)."""
    if _multi(group):
        dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    return counts


def join_count_distributed(canvas, xy_shard, count_fn=None, group=None) -> torch.Tensor:
    """COUNT of this rank's shard, then all_reduce: every rank ends with the global counts."""
    if count_fn is None:
        from . import join_count as count_fn
    counts = count_fn(canvas, xy_shard)
    return allreduce_counts(counts, group)


def _sizes(n: int, device, group=None) -> list[int]:
    world = dist.get_world_size(group)
    t = torch.tensor([n], dtype=torch.int64, device=device)
    sizes = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(sizes, t, group=group)
    return [int(s.item()) for s in sizes]


def gather_variable(t: torch.Tensor, dst: int = 0, group=None):
    """Gather 1-D tensors of different lengths to rank `dst` (rank order).  Sizes are
    all_gathered, then every other rank sends exactly its tensor to dst, which receives into
    one buffer of the total size.  Returns the concatenation on dst, None elsewhere."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    sizes = _sizes(t.numel(), t.device, group)
    if rank != dst:
        if t.numel():
            dist.send(t.contiguous(), dst=dist.get_global_rank(group, dst) if group is not None else dst, group=group)
        return None
    out = torch.empty(sum(sizes), dtype=t.dtype, device=t.device)
    offs = [sum(sizes[:r]) for r in range(world)]
    out[offs[rank]: offs[rank] + sizes[rank]] = t
    reqs = []
    for r in range(world):
        if r != rank and sizes[r]:
            src = dist.get_global_rank(group, r) if group is not None else r
            reqs.append(dist.irecv(out[offs[r]: offs[r] + sizes[r]], src=src, group=group))
    for q in reqs:
        q.wait()
    return out


def gather_pairs(point_ids: torch.Tensor, poly_ids: torch.Tensor, dst: int = 0, group=None):
    """Per-rank (global point id, polygon id) pairs -> all pairs on rank dst (order: by rank)."""
    a = gather_variable(point_ids, dst, group)
    b = gather_variable(poly_ids, dst, group)
    return (a, b) if a is not None else None


def join_pairs_distributed(canvas, xy_shard, point_id_base: int, pairs_fn=None, gather: bool = False, dst: int = 0,
                           group=None):
    """PAIRS of this rank's shard with global point ids.  Default: the shard's own pairs
    (sharded output, no exchange).  gather=True: all pairs on rank `dst` (None elsewhere)."""
    if pairs_fn is None:
        from . import join_pairs
        pairs_fn = lambda cv, xy, base: join_pairs(cv, xy, point_id_base=base)  # noqa: E731
    pt, pl = pairs_fn(canvas, xy_shard, point_id_base)
    if not gather or not _multi(group):
        return pt, pl
    return gather_pairs(pt, pl, dst, group)


def select_distributed(canvas, xy_shard, point_id_base: int, select_fn=None, gather: bool = False, dst: int = 0,
                       group=None):
    """SELECT of this rank's shard with global point ids (sharded by default, see above)."""
    if select_fn is None:
        from . import select
        select_fn = lambda cv, xy, base: select(cv, xy, point_id_base=base)  # noqa: E731
    ids = select_fn(canvas, xy_shard, point_id_base)
    if not gather or not _multi(group):
        return ids
    return gather_variable(ids, dst, group)


def canvas_checksums_agree(canvas, checksum_fn=None, group=None) -> bool:
    """Replicated-canvas check: every rank hashes its canvas (the canvas
    arrays on its device, spade_canvas_checksum) and the hashes are all_gathered and compared.
    True on every rank iff all ranks built bit-identical canvases."""
    if checksum_fn is None:
        from . import canvas_checksum as checksum_fn
    h = int(checksum_fn(canvas))
    if not _multi(group):
        return True
    dev = torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl" else torch.device("cpu")
    t = torch.tensor([h - (1 << 64) if h >= (1 << 63) else h], dtype=torch.int64, device=dev)
    hs = [torch.zeros_like(t) for _ in range(dist.get_world_size(group))]
    dist.all_gather(hs, t, group=group)
    return all(int(x.item()) == int(t.item()) for x in hs)


def all_gather_variable(t: torch.Tensor, group=None) -> torch.Tensor:
    """Concatenation (rank order) of 1-D tensors of different lengths, on every rank."""
    world = dist.get_world_size(group)
    sizes = _sizes(t.numel(), t.device, group)
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
      2. every rank picks the same circle (smallest with COUNT >= k) and selects its candidates
         (the circle's GLOBAL count bounds every shard's, so it is the selection's capacity);
      3. candidates all_gather'ed (about k in total), then sorted by (dist2, id): every rank
         holds the same top k.
    The per-step functions default to the CUDA path (knn_histogram / knn_radius / knn_select /
    knn_topk) and are injectable so the combine logic runs under gloo on CPU in the tests."""
    if hist_fn is None:
        from . import knn_histogram as hist_fn
    if radius_fn is None:
        from . import knn_radius as radius_fn
    if topk_fn is None:
        from . import knn_topk as topk_fn
    hist = hist_fn(xy_shard, q)
    if _multi(group):
        dist.all_reduce(hist, op=dist.ReduceOp.SUM, group=group)
    h = hist.cpu().numpy()
    if h[-1] > 0:
        raise ValueError(f"knn: {int(h[-1])} points outside [-2^30, 2^30)")
    r2, count = radius_fn(h, k)
    if select_fn is None:
        from . import knn_select
        ids, d2 = knn_select(xy_shard, q, r2, point_id_base=point_id_base, capacity=max(int(count), 0))
    else:
        ids, d2 = select_fn(xy_shard, q, r2, point_id_base)
    if _multi(group):
        ids = all_gather_variable(ids, group)
        d2 = all_gather_variable(d2, group)
    return topk_fn(ids, d2, k)
