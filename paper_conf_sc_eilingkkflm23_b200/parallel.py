"""Multi-GPU plumbing for the benchmark: one process per GPU, each an independent Cricket server endpoint
(no cross-GPU exchange exists on the memcpy path, so there is no data-path collective).
torch.distributed is used only to line the ranks up (barrier) and to reduce the timings: the job's time is
the max over ranks, its work the sum over ranks (weak scaling)."""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def rank_env() -> tuple[int, int, int]:
    """(world, rank, local_rank) from the torch.distributed.run environment."""
    return (int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")),
            int(os.environ.get("LOCAL_RANK", "0")))


def _reduce(x: float, op, device) -> float:
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=op)
    return float(t.item())


def max_over_ranks(x: float, device="cpu") -> float:
    return _reduce(x, dist.ReduceOp.MAX, device)


def sum_over_ranks(x: float, device="cpu") -> float:
    return _reduce(x, dist.ReduceOp.SUM, device)


def barrier(device=None):
    if device is not None and torch.cuda.is_available() and str(device).startswith("cuda"):
        torch.cuda.synchronize(device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.barrier()


def aggregate(units_local: float, seconds_local: float, device="cpu") -> dict:
    """Whole-job throughput: units processed by all ranks / the slowest rank's time."""
    t = max_over_ranks(seconds_local, device)
    u = sum_over_ranks(units_local, device)
    return {"seconds": t, "units": u, "per_second": u / t if t > 0 else 0.0}


def _cpulist(text: str) -> set[int]:
    cpus: set[int] = set()
    for part in text.strip().split(","):
        if not part:
            continue
        a, _, b = part.partition("-")
        cpus.update(range(int(a), int(b or a) + 1))
    return cpus


def bind_numa(device: int, sysfs: str = "/sys") -> dict:
    """Pins this process to the host cores of the NUMA node that `device` hangs off (SURVEY.md §8(d):
    rings sit on the GPU's NUMA node, so pinned buffers allocated afterwards are first-touched there and
    host-link traffic does not cross the socket interconnect).  Returns what was done, for the bench line."""
    p = torch.cuda.get_device_properties(device)
    bdf = f"{p.pci_domain_id:04x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
    try:
        node = int(open(f"{sysfs}/bus/pci/devices/{bdf}/numa_node").read().strip())
    except (OSError, ValueError):
        return {"pci": bdf, "numa_node": None}
    if node < 0:
        return {"pci": bdf, "numa_node": node}
    try:
        cpus = _cpulist(open(f"{sysfs}/devices/system/node/node{node}/cpulist").read())
        cpus &= os.sched_getaffinity(0)
        if cpus:
            os.sched_setaffinity(0, cpus)
    except OSError:
        cpus = set()
    return {"pci": bdf, "numa_node": node, "cores": len(cpus)}
