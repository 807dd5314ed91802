"""Drive a strings_workload.Workload through the C ABI (the public API a user calls).

Registers the tenants, submits every job (in the workload's submission order)
with its host buffers, waits for completion and collects the decision trace,
the outputs and per-job records.  No scheduling or kernel arithmetic happens
here: it is argument marshalling around libstrings_sched.so.
"""
from __future__ import annotations

import time
from dataclasses import dataclass, field
from typing import List, Optional

import numpy as np

import strings_workload as W

from . import strings as S


@dataclass
class RunResult:
    trace: List[str]
    outputs: List[List[np.ndarray]]
    infos: list
    stats: object
    wall_submit_to_drain_s: float
    status: int
    inputs: List[List[np.ndarray]] = field(default_factory=list)


def run_workload(wl: W.Workload, timing_mode: int = S.INJECTED, pinned: bool = True,
                 inputs: Optional[List[List[np.ndarray]]] = None, keep_inputs: bool = False,
                 trace_path: Optional[str] = None, physical_gpus: int = 0, kl_mode: int = 0,
                 slot_bytes: int = 0, torch_memory: bool = True, streams=None,
                 library_defaults: bool = False) -> RunResult:
    """library_defaults: pass the workload's config as written (A = 0, M = 0,
    joint_select = -1 ...) and let the library fill in its defaults, instead of
    the generator's resolved values."""
    cfg = wl.config.resolved()
    init_cfg = wl.config if library_defaults else cfg
    arenas = None
    if timing_mode != S.DECISIONS_ONLY and torch_memory:
        import torch                       # PyTorch provides the device memory (slot arenas)
        nphys = physical_gpus or torch.cuda.device_count()
        arenas = S.torch_arenas(cfg.num_gpus, min(nphys, cfg.num_gpus), cfg.admit_cap, slot_bytes)
        physical_gpus = len(arenas)
    S.init_from_config(init_cfg, timing_mode=timing_mode, trace_path=trace_path, physical_gpus=physical_gpus,
                       kl_mode=kl_mode, slot_bytes=slot_bytes, arenas=arenas, streams=streams)
    pinned_arrays = []
    try:
        for t in wl.tenants:
            S.register_tenant(t.weight, t.max_inflight)
        ins_all, outs_all = [], []
        dummy = np.zeros(16, dtype=np.uint8)       # decisions-only: buffers are never touched
        for i, spec in enumerate(wl.jobs):
            if timing_mode == S.DECISIONS_ONLY:
                ins_all.append([S.HostRef(dummy.ctypes.data, b) for b in spec.h2d_sizes()])
                outs_all.append([S.HostRef(dummy.ctypes.data, b) for b in spec.d2h_sizes()])
                continue
            if inputs is not None:
                src = inputs[i]
            else:
                src = W.job_inputs(spec)
            outs = []
            for shape, dt in W.job_output_shapes(spec):
                if pinned and timing_mode != S.DECISIONS_ONLY:
                    a = S.pinned_array(shape, dt)
                    pinned_arrays.append(a)
                else:
                    a = np.zeros(shape, dtype=dt)
                outs.append(a)
            if pinned and timing_mode != S.DECISIONS_ONLY:
                pins = []
                for a in src:
                    p = S.pinned_array(a.shape, a.dtype)
                    p[...] = a
                    pinned_arrays.append(p)
                    pins.append(p)
                src = pins
            ins_all.append(src)
            outs_all.append(outs)
        t0 = time.perf_counter()
        for i, spec in enumerate(wl.jobs):
            S.submit_spec(spec.tenant, spec, ins_all[i], outs_all[i])
        status = S.drain()
        wall = time.perf_counter() - t0
        tr = S.trace()
        infos = [S.job_info(i) for i in range(len(wl.jobs))]
        st = S.stats()
        outputs = [] if timing_mode == S.DECISIONS_ONLY else \
            [[np.array(o, copy=True) for o in outs] for outs in outs_all]
        kept = [[np.array(a, copy=True) for a in ins] for ins in ins_all] if keep_inputs else []
    finally:
        S.shutdown()
        for a in pinned_arrays:
            S.free_pinned(a)
        del arenas
    return RunResult(tr, outputs, infos, st, wall, status, kept)
