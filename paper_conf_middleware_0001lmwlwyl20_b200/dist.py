"""Multi-GPU sweep: candidates shard as c = rank (mod W); each
rank's fastt_sweep_best returns its lexicographically smallest
(makespan, index); the only exchange is an all_reduce(MIN) argmin over
torch.distributed (NCCL over NVLink on the GPU box, gloo in the CPU tests).

combine_best is a two-pass min -- first the makespan, then the smallest index
among ranks that hold that makespan -- so it is exact for any index range
(no bit packing limits) and ties resolve to the smallest global index (R3).
"""
from __future__ import annotations

import torch
import torch.distributed as dist

INT64_MAX = (1 << 63) - 1


def combine_best(best: torch.Tensor, group=None) -> torch.Tensor:
    """best: int64 tensor [makespan, index] (index -1 = none feasible),
    replaced in place by the global lexicographic minimum."""
    ms = best[0:1].clone()
    dist.all_reduce(ms, op=dist.ReduceOp.MIN, group=group)
    mine = torch.where((best[0:1] == ms) & (best[1:2] >= 0), best[1:2], torch.full_like(best[1:2], INT64_MAX))
    dist.all_reduce(mine, op=dist.ReduceOp.MIN, group=group)
    idx = torch.where(mine == INT64_MAX, torch.full_like(mine, -1), mine)
    best[0:1] = torch.where(idx >= 0, ms, torch.full_like(ms, INT64_MAX))
    best[1:2] = idx
    return best


def sweep_best_distributed(graph, gen, n_per_rank, flags=0, stream=None, group=None):
    """Global window [0, W*n_per_rank): rank r evaluates c = r + q*W."""
    W = dist.get_world_size(group) if dist.is_initialized() else 1
    r = dist.get_rank(group) if dist.is_initialized() else 0
    dev = torch.device("cuda", graph.device)
    out = torch.zeros(2, dtype=torch.int64, device=dev)
    graph.sweep_best(gen, r, n_per_rank, stride=W, flags=flags, stream=stream, out=out)
    if W > 1:
        combine_best(out, group)
    return int(out[0].item()), int(out[1].item())
