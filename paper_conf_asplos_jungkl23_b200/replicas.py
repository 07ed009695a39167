"""Multi-GPU = independent replicas.

DeepUM's path shares nothing between GPUs: each rank runs its own
oversubscribed trace (seed 3 + 1000 * rank), exec map, tables, residency and
host arena.  There is no data-path collective; torch.distributed (NCCL on the
GPU box, gloo in the CPU tests) carries only the start barrier and the
max-over-ranks timing reduction of the benchmark.
"""
from __future__ import annotations

from typing import Tuple

import torch


def replica_seed(base_seed: int, rank: int) -> int:
    return base_seed + 1000 * rank


def aggregate(total_ms: float, records: float, device=None) -> Tuple[float, float]:
    """(max over ranks of the timed region, sum over ranks of the work)."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(total_ms), float(records)
    dev = device if device is not None else torch.device("cpu")
    t = torch.tensor([float(total_ms)], dtype=torch.float64, device=dev)
    r = torch.tensor([float(records)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    dist.all_reduce(r, op=dist.ReduceOp.SUM)
    return float(t.item()), float(r.item())
