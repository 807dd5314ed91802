"""Static CUDA-runtime provisioning baseline (reading R-18).

One OS process per tenant (separate CUDA contexts, time-sliced, no MPS), a
static device choice, synchronous host<->device copies from pinned host
buffers, one plain kernel launch per job followed by a device synchronise --
what each tenant would do on its own with the CUDA runtime.  The tenant kernels
are the same device bodies the scheduler runs (launched stand-alone on the
whole GPU through strings_kernel_launch).

Device choice (SURVEY C-18):
  'mod'  -- tenant t on device t mod G (charitable: no two tenants collide
            unless there are more tenants than GPUs);
  'zero' -- every tenant on device 0, the SDK-style default pick (the paper's
            "static collisions").

Processes are spawned once per variant; every repeat starts from a barrier
after all contexts and buffers exist, so spawning and allocation are never
timed.  Like the Strings arm, a tenant's jobs share one pinned input and one
pinned output set (c_t = 1: a tenant's jobs never overlap; each job still
moves its own bytes each way).
"""
from __future__ import annotations

import multiprocessing as mp
import os
import statistics
import time
from typing import List


def _tenant_proc(t: int, dev: int, specs, repeats: int, barrier, out_q):
    import numpy as np
    import torch

    import strings_workload as W
    from paper_conf_sc_senguptagsp14_b200 import strings as S

    torch.cuda.set_device(dev)
    # one buffer set per distinct shape of the tenant's jobs (phase-changing tenants have up to 3)
    bufs = {}
    for spec in specs:
        key = (spec.kclass, spec.n, spec.m, spec.k)
        if key not in bufs:
            ins = [torch.from_numpy(a).pin_memory() for a in W.job_inputs(spec)]
            dins = [torch.empty_like(a, device="cuda") for a in ins]
            outs = [torch.empty(shape, dtype=getattr(torch, np.dtype(dt).name), device="cpu").pin_memory()
                    for shape, dt in W.job_output_shapes(spec)]
            douts = [torch.empty_like(o, device="cuda") for o in outs]
            bufs[key] = (ins, dins, outs, douts)
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream().cuda_stream
    for rep in range(repeats):
        barrier.wait()
        t0 = time.monotonic_ns()
        ends = []
        for spec in specs:
            ins, dins, outs, douts = bufs[(spec.kclass, spec.n, spec.m, spec.k)]
            for h, d in zip(ins, dins):
                d.copy_(h)                       # synchronous H2D (pinned)
            torch.cuda.synchronize()
            desc = S.make_desc(spec.kclass, n=spec.n, m=spec.m, k=spec.k, reps=spec.reps, alpha=spec.alpha,
                               seed=spec.seed)
            S.kernel_launch(dev, desc, [d.data_ptr() for d in dins], [d.data_ptr() for d in douts], ctas=0,
                            stream=stream)
            torch.cuda.synchronize()             # cudaDeviceSynchronize per job
            for h, d in zip(outs, douts):
                h.copy_(d)                       # synchronous D2H
            ends.append(time.monotonic_ns())
        out_q.put((rep, t, t0, time.monotonic_ns(), len(specs), ends))


def device_of(t: int, num_gpus: int, policy: str) -> int:
    return (t % num_gpus) if policy == "mod" else 0


def run_static(wl, num_gpus: int = 1, policy: str = "mod", repeats: int = 5) -> dict:
    """Time the workload under static provisioning; returns jobs/s (median over
    repeats, with min and max) and each tenant's mean completion latency.
    num_gpus = the physical GPUs the tenants are spread over ('mod')."""
    ctx = mp.get_context("spawn")
    by_tenant: List[list] = [[] for _ in wl.tenants]
    for s in wl.jobs:
        by_tenant[s.tenant].append(s)
    barrier = ctx.Barrier(len(by_tenant))
    q = ctx.Queue()
    procs = []
    for t, specs in enumerate(by_tenant):
        p = ctx.Process(target=_tenant_proc, args=(t, device_of(t, num_gpus, policy), specs, repeats, barrier, q),
                        daemon=True)
        p.start()
        procs.append(p)
    res = [q.get(timeout=1800) for _ in range(len(procs) * repeats)]
    for p in procs:
        p.join(timeout=120)
    spans, lats = [], []
    for rep in range(repeats):
        rr = [r for r in res if r[0] == rep]
        t0 = min(r[2] for r in rr)
        t1 = max(r[3] for r in rr)
        spans.append((t1 - t0) / 1e9)
        # mean completion latency per tenant (all jobs arrive at the common start t0)
        lats.append({r[1]: sum(e - t0 for e in r[5]) / max(1, len(r[5])) / 1e9 for r in rr})
    order = sorted(range(repeats), key=lambda i: spans[i])
    mid = order[len(order) // 2]
    span = spans[mid]
    vals = [len(wl.jobs) / s for s in spans]
    return {"value": len(wl.jobs) / span, "unit": "jobs/s", "span_s": span, "processes": len(by_tenant),
            "value_min": round(min(vals), 3), "value_max": round(max(vals), 3),
            "value_median": round(statistics.median(vals), 3),
            "spans_s": [round(x, 4) for x in spans],
            "mean_latency_s_by_tenant": {int(k): round(v, 6) for k, v in sorted(lats[mid].items())},
            "policy": f"tenant mod {num_gpus}" if policy == "mod" else "device 0 (every tenant)",
            "gpus_used": num_gpus if policy == "mod" else 1,
            "copies": "synchronous cudaMemcpy from pinned host memory", "repeats": repeats,
            "spawn": "one process per tenant, spawned once; each repeat starts at a barrier"}
