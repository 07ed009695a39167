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


def _reduce_device(device):
    """gloo reduces host tensors, NCCL device tensors."""
    import torch.distributed as dist
    if device is None or dist.get_backend() == "gloo":
        return torch.device("cpu")
    return device


def aggregate(total_ms: float, records: float, device=None) -> Tuple[float, float]:
    """(max over ranks of the timed region, sum over ranks of the work)."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(total_ms), float(records)
    dev = _reduce_device(device)
    t = torch.tensor([float(total_ms)], dtype=torch.float64, device=dev)
    r = torch.tensor([float(records)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    dist.all_reduce(r, op=dist.ReduceOp.SUM)
    return float(t.item()), float(r.item())


def aggregate_many(values, device=None, op="sum"):
    """Element-wise sum (or max) over ranks of a list of floats."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return [float(v) for v in values]
    t = torch.tensor([float(v) for v in values], dtype=torch.float64, device=_reduce_device(device))
    dist.all_reduce(t, op=dist.ReduceOp.SUM if op == "sum" else dist.ReduceOp.MAX)
    return [float(v) for v in t.tolist()]


def barrier():
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.barrier()


def local_cpus_of_gpu(index: int):
    """The host CPUs local to GPU `index` (its PCI device's local_cpulist in
    sysfs), or None when unknown.  One replica per GPU is bound to them so that
    its pinned host arena and its driver threads sit on the GPU's NUMA node
    (numactl --cpunodebind/--membind equivalent)."""
    try:
        p = torch.cuda.get_device_properties(index)
        bus = "%04x:%02x:%02x.0" % (int(getattr(p, "pci_domain_id", 0)), int(p.pci_bus_id), int(p.pci_device_id))
    except Exception:
        return None
    for path in ("/sys/bus/pci/devices/%s/local_cpulist" % bus,):
        try:
            txt = open(path).read().strip()
        except OSError:
            continue
        cpus = set()
        for part in txt.split(","):
            if "-" in part:
                a, b = part.split("-")
                cpus.update(range(int(a), int(b) + 1))
            elif part:
                cpus.add(int(part))
        return sorted(cpus) or None
    return None


def bind_to_gpu_node(index: int):
    """Bind this process to the CPUs local to GPU `index` (first-touch then
    places its host allocations on that NUMA node).  Returns a report dict."""
    import os
    try:
        cpus = local_cpus_of_gpu(index)
    except Exception as e:  # never fatal: binding is a placement hint
        return {"bound": False, "why": "lookup failed: %s" % e}
    if not cpus:
        return {"bound": False, "why": "no sysfs local_cpulist for the GPU"}
    try:
        avail = os.sched_getaffinity(0)
        use = [c for c in cpus if c in avail]
        if not use:
            return {"bound": False, "why": "GPU-local CPUs outside this process's allowed set"}
        os.sched_setaffinity(0, use)
        return {"bound": True, "cpus": "%d-%d" % (min(use), max(use)), "n_cpus": len(use)}
    except OSError as e:
        return {"bound": False, "why": str(e)}
