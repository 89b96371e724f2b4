"""Multi-GPU sharding of the replay.

Traces are independent, so the data path has no collective: rank r of G
replays the contiguous global trace-id range [r*N/G, (r+1)*N/G) that it
generates itself on its own GPU (the counter-based generator keys every trace
by its global id).  The only exchange is the final reduction of the
per-policy statistics record (§8(a) row a7): SUM over the u64 sums and the
u32 flag counters, MAX over the two u32 maxima, and SUM of the per-range
digest vector (ranges are disjoint, so SUM = gather).  These run as NCCL
all-reduces over NVLink on views of the tensors the kernels wrote — no host
staging, no repacking kernels.  With the gloo backend the same code runs on
CPU tensors (tests).
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(total: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous [lo, hi) of global trace ids owned by `rank`."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError("bad rank/world")
    return total * rank // world, total * (rank + 1) // world


def reduce_stats(stats: torch.Tensor, group=None) -> torch.Tensor:
    """All-reduce one convgpu_stats_t record (int64[12], 96 B) in place.

    Layout (include/convgpu.h): u64[0..6] sums; u32[14] max_makespan,
    u32[15] max_peak_reserved; u32[16..23] flag counts."""
    if stats.dtype != torch.int64 or stats.numel() != 12 or not stats.is_contiguous():
        raise ValueError("stats must be a contiguous int64[12] convgpu_stats_t")
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        w32 = stats.view(torch.int32)
        dist.all_reduce(stats[0:7], op=dist.ReduceOp.SUM, group=group)   # u64 sums, mod 2^64
        dist.all_reduce(w32[14:16], op=dist.ReduceOp.MAX, group=group)   # values < 2^26
        dist.all_reduce(w32[16:24], op=dist.ReduceOp.SUM, group=group)
    return stats


def reduce_stats_block(block: torch.Tensor, group=None) -> torch.Tensor:
    """All-reduce m convgpu_stats_t records at once (int64[m, 12], e.g. the
    four policies of one bench step) in place with two collectives instead of
    3m: one SUM over the whole block as int64 (right for the seven u64 sums and
    for the eight u32 flag counters, whose pairs share an int64 word: a
    counter is at most the number of traces, < 2^32, so no carry crosses
    into its neighbour) and one MAX over the block viewed as int32, whose
    words 14 / 15 of each record are the two u32 maxima (< 2^31)."""
    if (block.dtype != torch.int64 or block.dim() != 2 or block.shape[1] != 12
            or not block.is_contiguous()):
        raise ValueError("block must be a contiguous int64[m, 12] array of convgpu_stats_t")
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        mx = block.view(torch.int32).clone()
        dist.all_reduce(block, op=dist.ReduceOp.SUM, group=group)
        dist.all_reduce(mx, op=dist.ReduceOp.MAX, group=group)
        block.view(torch.int32)[:, 14:16] = mx[:, 14:16]
    return block


def reduce_range_digests(rd: torch.Tensor, group=None) -> torch.Tensor:
    """SUM-all-reduce a per-range digest vector (int64, mod 2^64) in place."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(rd, op=dist.ReduceOp.SUM, group=group)
    return rd


def max_over_ranks(x: float, device) -> float:
    """Max of a host scalar over ranks (timing: the slowest rank decides)."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
