"""Host-side multi-GPU plumbing over torch.distributed.

The data path runs in libspg: flop-balanced split points are computed on each rank's GPU
(`spg_split_points` / inside `spg_spgemm_symbolic` of a dist handle), B is replicated by NCCL
broadcast (`spg_broadcast_csr`), C blocks are gathered by `spg_allgatherv_c`.  This module only
bootstraps the NCCL communicator from a torch process group and provides the host-side pieces
the benchmark and tests share: row ranges, max-over-ranks timing, and a reference
`allgatherv` of C blocks over the process group (used to check the NCCL path, and to exercise
the partition/rebase bookkeeping with gloo on CPU).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def rank_rows(splits, rank: int):
    """Rows [s_rank, s_rank+1) owned by `rank` (splits: s_0 = 0 <= ... <= s_P = M)."""
    s = np.asarray(splits)
    return int(s[rank]), int(s[rank + 1])


def max_over_ranks(x: float, group=None, device=None) -> float:
    """Max of a per-rank scalar over the group (step time of a multi-GPU step)."""
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def create_dist_handle(device: int, stream, dtype, group=None):
    """spg_create_dist with the NCCL unique id broadcast over `group` (any backend)."""
    from .binding import spg_create_dist, spg_get_unique_id
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    obj = [spg_get_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return spg_create_dist(device, stream, dtype, obj[0], rank, world)


def allgatherv_c(row_ptr_local, col_local, val_local, splits, group=None):
    """Reference allgatherv of per-rank C row blocks (numpy in, numpy out).

    row_ptr_local starts at 0 for the rank's first row (the ABI's local convention); the
    result is the full C with global int64 row offsets — rank r's offsets are rebased by the
    nnz of ranks < r, exactly what spg_allgatherv_c's rebase kernel does.
    """
    world = dist.get_world_size(group)
    nnz = torch.tensor([int(row_ptr_local[-1])], dtype=torch.int64)
    sizes = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(sizes, nnz, group=group)
    sizes = [int(s.item()) for s in sizes]
    off = np.concatenate([[0], np.cumsum(sizes)]).astype(np.int64)
    blocks = [None] * world
    dist.all_gather_object(blocks, (np.asarray(row_ptr_local, np.int64), np.asarray(col_local, np.int32),
                                    np.asarray(val_local)), group=group)
    M = int(np.asarray(splits)[-1])
    rp = np.zeros(M + 1, np.int64)
    for r in range(world):
        s0, s1 = rank_rows(splits, r)
        rp[s0:s1] = blocks[r][0][: s1 - s0] + off[r]
    rp[M] = off[-1]
    col = np.concatenate([b[1] for b in blocks]) if off[-1] else np.zeros(0, np.int32)
    val = np.concatenate([b[2] for b in blocks]) if off[-1] else np.zeros(0, np.float64)
    return rp, col, val
