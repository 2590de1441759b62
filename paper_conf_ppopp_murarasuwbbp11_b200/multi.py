"""Multi-GPU decompression: one global order, contiguous shards, one broadcast.

Evaluation is embarrassingly parallel over query points (Sec. 4.3): every query costs
exactly T(d, n) terms, so a static partition into equal ranges balances perfectly -- the paper's "static
workload distribution" (L51).  The path on P ranks:

1. rank ``src`` compresses (hierarchizes); ONE broadcast of the surplus array (NCCL over NVLink/NVSwitch
   on B200, 1.02 GB at cfg3; gloo in the CPU tests) replicates it -- the path's only collective;
2. every rank orders the WHOLE batch along the Morton curve (``sg_sfc_order``: a deterministic stable
   radix sort, so all ranks obtain the same permutation without communicating, in ~ms);
3. rank r evaluates the contiguous range ``partition(m, P, r)`` of that global order
   (``sg_evaluate_ordered``).  Ranges of one global order keep every rank's warps as compact as on one
   GPU; per-rank local sorts of index slices would not (6.95 vs 4.86 sectors per gather).

Outputs stay sharded: rank r's result vector holds the values of its range's queries (at their input
positions).  Every query's value is bitwise the same whichever rank evaluates it (the per-query
arithmetic order is fixed by the enumeration), so the union over ranks equals one-GPU evaluation.
"""
from __future__ import annotations


def partition(m: int, world: int, rank: int) -> tuple[int, int]:
    """(first, count) of rank's contiguous range of an m-query order: sizes differ by at most one."""
    if m < 0 or world < 1 or not 0 <= rank < world:
        raise ValueError(f"bad partition arguments m={m} world={world} rank={rank}")
    q, r = divmod(m, world)
    first = rank * q + min(rank, r)
    return first, q + (1 if rank < r else 0)


def replicate_surpluses(alpha, src: int = 0, group=None):
    """Broadcast the surplus array from ``src`` to every rank, in place (north_star: "replicated with one
    NCCL broadcast").  ``alpha`` is a contiguous tensor on the rank's device (CUDA for NCCL, CPU or CUDA
    for gloo)."""
    import torch.distributed as dist
    if not alpha.is_contiguous():
        raise ValueError("alpha must be contiguous")
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.broadcast(alpha, src=src, group=group)
    return alpha


def evaluate_distributed(grid, alpha, x, group=None, src: int = 0, out=None, perm=None, broadcast: bool = True):
    """Evaluate this rank's shard of the batch ``x`` (the WHOLE batch, identical on every rank).

    ``alpha`` is broadcast from ``src`` first (skip with ``broadcast=False`` when it is already
    replicated); ``perm`` may be passed to reuse an order computed earlier.  Returns
    ``(y, perm, first, count)``: ``y`` (whole-batch length, input order) holds this rank's values at the
    positions ``perm[first:first+count]``; other entries are left as they were (zeros if ``out`` is None).
    """
    import torch.distributed as dist
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    if broadcast:
        replicate_surpluses(alpha, src=src, group=group)
    if perm is None:
        perm = grid.sfc_order(x)
    first, count = partition(x.shape[0], world, rank)
    y = grid.evaluate_ordered(alpha, x, perm, first, count, out=out)
    return y, perm, first, count


def evaluate_sharded_grid(grid, alpha_part, x, group=None, out=None):
    """Evaluate a grid whose surpluses are sharded across the ranks (grids larger than
    one GPU): rank r holds only part r of P (``grid.part_bounds(P, r)``: a contiguous, work-balanced range of
    the layout) and evaluates that part's share of f_s at EVERY query of the batch ``x``; one all-reduce
    (sum) of the m results -- the path's only collective, m values instead of the N surpluses -- gives
    every rank f_s(x).  Parts are summed in rank order by the collective, so the result equals one-GPU
    evaluation up to rounding (not bitwise)."""
    import torch.distributed as dist
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    y = grid.evaluate_part(alpha_part, world, rank, x, out=out)
    if world > 1:
        dist.all_reduce(y, op=dist.ReduceOp.SUM, group=group)
    return y


def checksum(t) -> int:
    """Order-sensitive 64-bit checksum of a tensor's bytes (for replication checks)."""
    import numpy as np
    raw = t.detach().cpu().contiguous().view(-1).numpy().view(np.uint8)
    b = np.concatenate([raw, np.zeros(-raw.size % 8, dtype=np.uint8)]).view(np.uint64)
    w = (np.arange(b.size, dtype=np.uint64) * np.uint64(0x9E3779B97F4A7C15)) | np.uint64(1)
    return int(np.bitwise_xor.reduce(b * w)) if b.size else 0
