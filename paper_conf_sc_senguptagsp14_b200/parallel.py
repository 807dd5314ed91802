"""Multi-GPU plumbing: one process per GPU, placement-only sharding.

Tenants are independent, so scaling across the GPUs of a box is placement
only: there is no data-path collective and no NCCL on the
hot path.  Two deployment shapes are supported:

* node mode -- one process owns G GPUs and the library's level-1 balancer
  places every job on one of them (``strings_init(num_gpus=G)``); this is the
  paper's design (one GPU affinity mapper per node);
* rank mode -- ``torchrun`` starts one process per GPU; each rank runs its own
  library instance on its own GPU over its shard of the tenants (weak scaling).

While the persistent dispatcher kernel is resident it owns every SM, so rank
coordination (barriers, max-over-ranks timing) must not launch device work or
synchronise the device: it goes through a CPU (gloo) group.
"""
from __future__ import annotations

import os
from dataclasses import dataclass
from typing import List, Optional


@dataclass
class RankInfo:
    rank: int
    world: int
    local_rank: int
    local_world: int = 1          # ranks on this node (torchrun's LOCAL_WORLD_SIZE)


def rank_info() -> RankInfo:
    world = int(os.environ.get("WORLD_SIZE", "1"))
    return RankInfo(int(os.environ.get("RANK", "0")), world,
                    int(os.environ.get("LOCAL_RANK", os.environ.get("RANK", "0"))),
                    int(os.environ.get("LOCAL_WORLD_SIZE", str(world))))


def isolate_gpu(info: RankInfo) -> None:
    """Make this rank's GPU the only visible one (must run before CUDA init).
    The rank takes the local_rank-th entry of an inherited CUDA_VISIBLE_DEVICES
    list (so a launcher that hands out e.g. "4,5,6,7" is respected), else the
    device with index local_rank."""
    if info.world > 1:
        os.environ["CUDA_VISIBLE_DEVICES"] = physical_gpu(info)
        if shared_gpu_test():
            # every rank on the first device, each dispatcher on its own share of the SMs
            os.environ.setdefault("STRINGS_SM_LIMIT", str(148 // info.world))
            # processes sharing a GPU time-slice their persistent kernels (separate
            # contexts, no MPS): a copy-partition op waits for its context's slice
            # (2 ranks: 1136-1193 jobs/s with copy engines only, 680-700 with the
            # copy partition), so the shared-GPU test keeps every copy on the engines
            os.environ.setdefault("STRINGS_COPY_CTAS", "0")


def shared_gpu_test() -> bool:
    """STRINGS_BENCH_SHARE_GPU=1: all ranks share the first visible GPU (a test of
    the multi-rank plumbing on a 1-GPU box; NCCL refuses two ranks per device, so
    the default group is gloo).  Never used for reported numbers."""
    return os.environ.get("STRINGS_BENCH_SHARE_GPU") == "1"


def physical_gpu(info: RankInfo) -> str:
    """The device id this rank uses, as the launcher numbers devices."""
    vis = [d.strip() for d in os.environ.get("STRINGS_INHERITED_CVD", os.environ.get("CUDA_VISIBLE_DEVICES", ""))
           .split(",") if d.strip()]
    os.environ.setdefault("STRINGS_INHERITED_CVD", ",".join(vis))
    if shared_gpu_test():
        return vis[0] if vis else "0"
    if vis and info.local_rank < len(vis):
        return vis[info.local_rank]
    return str(info.local_rank)


def bind_to_gpu_numa_node(gpu_id: str) -> dict:
    """Restrict this process (and the library threads it will start) to the CPUs
    of the NUMA node the GPU hangs off, so pinned buffers are first-touched on
    that node and the copy engines DMA without crossing the socket link (SURVEY
    §8(e): host DRAM and PCIe root complexes are shared).  No-op when the node
    cannot be determined; returns what was done."""
    import subprocess
    try:
        bus = subprocess.run(["nvidia-smi", f"--id={gpu_id}", "--query-gpu=pci.bus_id", "--format=csv,noheader"],
                             capture_output=True, text=True, timeout=30).stdout.strip().splitlines()[0]
        dom, rest = bus.split(":", 1)
        sysfs = f"/sys/bus/pci/devices/{dom[-4:]}:{rest}".lower()
        with open(sysfs + "/local_cpulist") as f:
            spec = f.read().strip()
        with open(sysfs + "/numa_node") as f:
            node = int(f.read().strip())
        cpus = set()
        for part in spec.split(","):
            a, _, b = part.partition("-")
            cpus.update(range(int(a), int(b or a) + 1))
        allowed = os.sched_getaffinity(0)
        use = cpus & allowed
        if not use or use == allowed:
            return {"numa_node": node, "cpus": len(allowed), "bound": False}
        os.sched_setaffinity(0, use)
        return {"numa_node": node, "cpus": len(use), "bound": True}
    except Exception as e:  # noqa: BLE001 - best effort
        return {"bound": False, "why": type(e).__name__}


def init_groups(info: RankInfo, device_backend: Optional[str] = "nccl", timeout_s: Optional[float] = None):
    """Default process group (NCCL when a GPU is present) plus a gloo group for
    host-side coordination.  Returns the gloo group (None for world == 1)."""
    if info.world == 1:
        return None
    import datetime

    import torch
    import torch.distributed as dist
    kw = {"timeout": datetime.timedelta(seconds=timeout_s)} if timeout_s else {}
    if device_backend == "nccl" and torch.cuda.is_available() and not shared_gpu_test():
        torch.cuda.set_device(0)
        dist.init_process_group("nccl", device_id=torch.device("cuda:0"), **kw)
        return dist.new_group(backend="gloo", **kw)
    dist.init_process_group("gloo", **kw)
    return dist.group.WORLD


def node_mode(info: RankInfo, group, work):
    """Node mode under a one-process-per-GPU launcher (torchrun): rank 0 runs
    `work(group)`, which owns every GPU of the node through the library's
    level-1 balancer and may call max_over_ranks(group, x) exactly
    once; the other ranks do no work (jobs are independent: no data-path
    collective), contribute 0 to that max and wait.  Returns work's result on
    rank 0, None elsewhere."""
    if info.rank == 0:
        out = work(group)
    else:
        max_over_ranks(group, 0.0)
        out = None
    barrier(group)
    return out


def barrier(group) -> None:
    if group is not None:
        import torch.distributed as dist
        dist.barrier(group=group)


def max_over_ranks(group, x: float) -> float:
    """Max over ranks of a host-side float (device timings are taken on each
    rank with CUDA events, then reduced here)."""
    if group is None:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def sum_over_ranks(group, x: float) -> float:
    if group is None:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return float(t.item())


def copy_threads_per_rank(info: RankInfo) -> int:
    """PMT staging threads for one rank when several ranks run on one node: the
    CPUs this rank may use, shared by the node's ranks bound to the same CPUs
    (all local ranks when the NUMA binding was a no-op), minus the engine and
    caller threads; at most the library's default of 12."""
    cpus = len(os.sched_getaffinity(0))
    total = max(cpus, os.cpu_count() or cpus)
    sharing = max(1, round(info.local_world * cpus / total))   # ranks bound to these same CPUs
    return max(2, min(12, cpus // sharing - 2))


def gather_over_ranks(group, xs: List[float]) -> List[float]:
    """Concatenation of every rank's list (rank order), e.g. per-tenant fairness
    inputs, so whole-job metrics (Jain over all N x 16 tenants) are computed once."""
    if group is None:
        return list(xs)
    import torch.distributed as dist
    out = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, list(xs), group=group)
    return [x for part in out for x in part]


def jain(xs: List[float]) -> float:
    """Jain's index (Eq. 3, reading R-2): (sum x)^2 / (n sum x^2), in [1/n, 1]."""
    return sum(xs) ** 2 / (len(xs) * sum(x * x for x in xs)) if xs else 1.0


def shard_tenants(num_tenants: int, world: int, rank: int) -> List[int]:
    """Tenants of this rank under strong scaling (round robin, like GRR)."""
    return [t for t in range(num_tenants) if t % world == rank]
