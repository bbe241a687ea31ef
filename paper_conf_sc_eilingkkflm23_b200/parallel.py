"""Multi-GPU plumbing for the benchmark: one process per GPU, each an independent Cricket server endpoint
(no cross-GPU exchange exists on the memcpy path, so there is no data-path collective and no
NCCL: BASELINE.json north_star).  torch.distributed with the CPU `gloo` backend only lines the ranks up
(barrier) and reduces the timings: the job's time is the max over ranks, its work the sum over ranks (weak
scaling); host-link rooflines are measured by every rank at once after a barrier and gathered."""
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


def init(world: int) -> bool:
    """Joins the job's process group (gloo, CPU) when there is more than one rank; no NCCL anywhere."""
    if world > 1 and not (dist.is_available() and dist.is_initialized()):
        dist.init_process_group("gloo")
        return True
    return False


def gather(obj) -> list:
    """Every rank's `obj`, in rank order (a list of one without a process group)."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return [obj]
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, obj)
    return out


def link_aggregate(per_rank: list[dict], keys=("ce_h2d_gbs", "ce_d2h_gbs", "ce_bidir_gbs")) -> dict:
    """Host-link peaks measured by all ranks at once (each rank's own GPU, concurrently): per rank and summed.
    The sum is the job's host-link roofline (PCIe switch uplinks and host memory are shared, so it can be less
    than N x one GPU alone)."""
    return {"per_rank": per_rank, "aggregate": {k: round(sum(r[k] for r in per_rank), 2) for k in keys},
            "ranks": len(per_rank)}


def link_bound_frac(per_rank_link: list[dict], per_rank_wire: list[tuple[int, int]], step_s: float) -> dict:
    """The job's e2e host-link fraction: every rank moves its own wire bytes (in, out) over its own link at the
    concurrently measured rate; the job can finish no sooner than its slowest rank's link-bound time."""
    bounds = [max(wi / l["ce_h2d_gbs"], wo / l["ce_d2h_gbs"], (wi + wo) / l["ce_bidir_gbs"]) / 1e9
              for l, (wi, wo) in zip(per_rank_link, per_rank_wire)]
    b = max(bounds)
    return {"bound_ms": round(b * 1e3, 3), "frac": round(b / step_s, 4), "per_rank_bound_ms": [round(x * 1e3, 3)
                                                                                                for x in bounds]}
