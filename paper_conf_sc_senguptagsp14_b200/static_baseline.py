"""Static CUDA-runtime provisioning baseline (reading R-18).

One OS process per tenant (separate CUDA contexts, time-sliced, no MPS), a
static device choice (tenant mod G, or device 0), synchronous host<->device
copies from pinned host buffers, one plain kernel launch per job followed by a
device synchronise -- what each tenant would do on its own with the CUDA
runtime.  The tenant kernels are the same device bodies the scheduler runs
(launched stand-alone on the whole GPU through strings_kernel_launch).
"""
from __future__ import annotations

import multiprocessing as mp
import os
import time
from typing import List


def _tenant_proc(t: int, dev: int, specs, barrier, out_q, visible: str):
    if visible is not None:
        os.environ["CUDA_VISIBLE_DEVICES"] = visible
    import numpy as np
    import torch

    import strings_workload as W
    from paper_conf_sc_senguptagsp14_b200 import strings as S

    torch.cuda.set_device(dev)
    jobs = []
    for spec in specs:
        ins = [torch.from_numpy(a).pin_memory() for a in W.job_inputs(spec)]
        dins = [torch.empty_like(a, device="cuda") for a in ins]
        outs = [torch.empty(shape, dtype=getattr(torch, np.dtype(dt).name), device="cpu").pin_memory()
                for shape, dt in W.job_output_shapes(spec)]
        douts = [torch.empty_like(o, device="cuda") for o in outs]
        jobs.append((spec, ins, dins, outs, douts))
    torch.cuda.synchronize()
    barrier.wait()
    t0 = time.monotonic_ns()
    ends = []
    for spec, ins, dins, outs, douts in jobs:
        for h, d in zip(ins, dins):
            d.copy_(h)                       # synchronous H2D (pinned)
        torch.cuda.synchronize()
        desc = S.make_desc(spec.kclass, n=spec.n, m=spec.m, k=spec.k, reps=spec.reps, alpha=spec.alpha,
                           seed=spec.seed)
        S.kernel_launch(dev, desc, [d.data_ptr() for d in dins], [d.data_ptr() for d in douts], ctas=0,
                        stream=torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()             # cudaDeviceSynchronize per job
        for h, d in zip(outs, douts):
            h.copy_(d)                       # synchronous D2H
        ends.append(time.monotonic_ns())
    t1 = time.monotonic_ns()
    out_q.put((t, t0, t1, len(jobs), ends))


def run_static(wl, num_gpus: int = 1, policy: str = "mod", repeats: int = 1) -> dict:
    """Time the workload under static provisioning; returns jobs/s and span.

    policy 'mod': tenant t on device t mod G (charitable); 'zero': all on device 0.
    All tenants start together (barrier after every context and buffer exists).
    """
    ctx = mp.get_context("spawn")
    by_tenant: List[list] = [[] for _ in wl.tenants]
    for s in wl.jobs:
        by_tenant[s.tenant].append(s)
    spans, lats = [], []
    for _ in range(repeats):
        barrier = ctx.Barrier(len(by_tenant))
        q = ctx.Queue()
        procs = []
        for t, specs in enumerate(by_tenant):
            dev = (t % num_gpus) if policy == "mod" else 0
            p = ctx.Process(target=_tenant_proc, args=(t, dev, specs, barrier, q, None), daemon=True)
            p.start()
            procs.append(p)
        res = [q.get(timeout=900) for _ in procs]
        for p in procs:
            p.join(timeout=120)
        t0 = min(r[1] for r in res)
        t1 = max(r[2] for r in res)
        spans.append((t1 - t0) / 1e9)
        # mean completion latency per tenant (all jobs arrive at the common start t0)
        lat = {r[0]: sum(e - t0 for e in r[4]) / max(1, len(r[4])) / 1e9 for r in res}
        lats.append(lat)
    order = sorted(range(len(spans)), key=lambda i: spans[i])
    mid = order[len(order) // 2]
    span = spans[mid]
    return {"value": len(wl.jobs) / span, "unit": "jobs/s", "span_s": span, "processes": len(by_tenant),
            "spans_s": [round(x, 4) for x in spans],
            "mean_latency_s_by_tenant": {int(k): round(v, 6) for k, v in sorted(lats[mid].items())},
            "policy": f"tenant mod {num_gpus}" if policy == "mod" else "device 0",
            "copies": "synchronous cudaMemcpy from pinned host memory", "repeats": repeats}
