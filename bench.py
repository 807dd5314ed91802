#!/usr/bin/env python
"""Benchmark: tenant jobs/sec of the Strings scheduler hot path on B200.

Workload (BASELINE.json configs[1], the single-GPU config):
C2 = 16 tenants (8 GEMM 256^3 R=64 + 8 XFER 2^24 u32), 8 jobs each, DTF
placement (joint selection), PS dispatch, MEASURED timing.  One "step" = the
whole hot path (submit -> balancer -> H2D -> persistent-kernel KL -> D2H ->
completion) over the 128 jobs of one C2 batch.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]

N > 1 runs under torchrun, one process per GPU; tenants are independent, so
each rank runs its own C2 batch on its own GPU (weak scaling, no collective
on the data path; rank timings are combined with a max over a CPU group).

JSON line keys beyond the base contract:
  roofline         dominant resource of the step = the host link (copy engines)
  overlapped_roofline   T*_d / span per SURVEY.md §8(d) with the measured peaks
  kernel_rooflines tenant kernels timed stand-alone (HBM GB/s, tensor TFLOP/s)
  static_baseline  one process per tenant, synchronous copies (reading R-18)
  cpu_baseline     the oracle (oracle/) on a bounded sample, on the host cores
"""
from __future__ import annotations

import argparse
import dataclasses
import json
import os
import statistics
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "tenant jobs/sec (8xB200) vs static CUDA provisioning; Jain fairness"
# The paper's headline ratios, quoted with their hardware as context only.
PAPER_CONTEXT = {
    "weighted_speedup_vs_cuda_runtime": {"PS": 6.41, "DTF": 8.06, "MBF": 8.70},
    "fairness_gain_vs_cuda_runtime": "13% (TFS-Strings, average Jain 91%)",
    "hardware": "2 nodes x 2 Fermi GPUs (Quadro 2000/4000, Tesla C2050/C2070), CUDA 5.0, 4-GPU supernode "
                "over GigE; CUDA SDK/Rodinia app pairs",
    "citations": "PAPER.md L29, L43, L879, L957, L1155",
    "note": "relative figures on other hardware and workloads: context, not a target (vs_baseline is null)"}


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=8)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="strings", choices=["strings", "reference"])
    p.add_argument("--jobs-per-tenant", type=int, default=8)
    p.add_argument("--no-static", action="store_true")
    p.add_argument("--no-kernels", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--kl-mode", type=int, default=0, help="0 persistent dispatcher, 1 per-job launches (ncu)")
    p.add_argument("--trace-out", default=None)
    p.add_argument("--static-repeats", type=int, default=5)
    p.add_argument("--awake-budget", type=int, default=0, help="A (0 = config default)")
    p.add_argument("--admit-cap", type=int, default=0, help="M (0 = config default)")
    p.add_argument("--partitions", type=int, default=0, help="P (0 = config default)")
    p.add_argument("--device-policy", type=int, default=-1, help="0 FIFO, 1 LAS, 2 PS (-1 = config)")
    p.add_argument("--balancer", type=int, default=-1, help="balancer id (-1 = config)")
    p.add_argument("--config-repeats", type=int, default=5, help="timed runs per config and seed in --configs")
    p.add_argument("--config-seeds", default="1", help="--configs: workload seeds, comma-separated (SURVEY: 1-5)")
    p.add_argument("--config-static", action="store_true", help="--configs: add static baselines")
    p.add_argument("--baseline-config-static", action="store_true",
                   help="N > 1: also time static provisioning on the BASELINE config")
    p.add_argument("--no-baseline-config", action="store_true",
                   help="N > 1: skip the BASELINE config whose G equals N (C1/C3/C5)")
    p.add_argument("--configs", action="store_true",
                   help="run BASELINE configs C1-C5 at full size (node mode, logical devices if G > GPUs)")
    p.add_argument("--fig2", action="store_true",
                   help="Fig. 2 analogue: N identical requests sequential vs co-resident vs separate contexts")
    p.add_argument("--open-loop", action="store_true",
                   help="C4 open loop: jobs submitted at their Eq. (4) arrival times; p50/p99 latency per "
                   "priority class, LAS+GUF vs arrival-order GMin+FIFO; not the driver line")
    p.add_argument("--open-loop-config", default="C4", choices=["C4", "C4c"],
                   help="C4c: the admission-contention variant (rho = 2, c_t = 4, M = 4)")
    p.add_argument("--open-loop-dilate", type=float, default=0.0,
                   help="arrival-time dilation (0 = logical devices per physical GPU, so the offered load "
                   "per physical host link is the config's rho)")
    p.add_argument("--sweep", action="store_true",
                   help="policy comparison on C2 (device policies x balancers) vs static; not the driver line")
    return p.parse_args()


# ----------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        # nvidia-smi --id: an index, bus id or UUID, or a list of them (node mode: every GPU used)
        self.index = ",".join(str(i) for i in index) if isinstance(index, (list, tuple)) else index
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except FileNotFoundError:
            self.p = None
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        if self.p:
            self.p.terminate()
            self.p.wait(timeout=10)

    def summary(self) -> dict:
        self.f.seek(0)
        rows = [r.split(",") for r in self.f.read().strip().splitlines() if r.strip()]
        sm = [float(r[1]) for r in rows if len(r) > 8 and r[1].strip().replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if len(r) > 8 and r[2].strip().replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            if len(r) > 8:
                for n, v in zip(names, r[5:9]):
                    if v.strip().lower() == "active":
                        reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(rows)}


# ------------------------------------------------------------- peaks
def measured_peaks() -> dict:
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return {"hbm_gbs": d["hbm_gbs"], "bf16_tflops": d["bf16_tflops"],
                "bf16_tflops_sustained": d.get("bf16_tflops_sustained"), "source": "MEASURED_PEAKS.json"}
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
            "source": "fallback (B200_PROFILING.md)"}


def host_link_peaks(torch, nbytes=256 << 20, iters=8) -> dict:
    """Pinned H2D, D2H and concurrent bidirectional copy bandwidth (GB/s),
    plain cudaMemcpyAsync through torch on dedicated streams."""
    h_in = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    h_out = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d_a = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d_b = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def timed(fn):
        best = None
        for _ in range(iters + 1):
            torch.cuda.synchronize()
            t = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            dt = time.perf_counter() - t
            best = dt if best is None else min(best, dt)
        return best

    def h2d():
        with torch.cuda.stream(s1):
            d_a.copy_(h_in, non_blocking=True)

    def d2h():
        with torch.cuda.stream(s2):
            h_out.copy_(d_b, non_blocking=True)

    def both():
        h2d()
        d2h()
    r = {"h2d_gbs": nbytes / timed(h2d) / 1e9, "d2h_gbs": nbytes / timed(d2h) / 1e9}
    r["bidir_gbs"] = 2 * nbytes / timed(both) / 1e9
    del h_in, h_out, d_a, d_b
    return r


def host_link_concurrent(torch, ngpu: int, nbytes=256 << 20, iters=8) -> dict:
    """H2D + D2H copies on every one of `ngpu` GPUs at once (the
    host's DRAM and PCIe root complexes are shared): aggregate GB/s and the
    per-GPU share, the link peak each device's T*_d uses in node mode."""
    res = []
    for g in range(ngpu):
        with torch.cuda.device(g):
            res.append((torch.empty(nbytes, dtype=torch.uint8).pin_memory(),
                        torch.empty(nbytes, dtype=torch.uint8).pin_memory(),
                        torch.empty(nbytes, dtype=torch.uint8, device=f"cuda:{g}"),
                        torch.empty(nbytes, dtype=torch.uint8, device=f"cuda:{g}"),
                        torch.cuda.Stream(device=g), torch.cuda.Stream(device=g)))
    best = None
    for _ in range(iters + 1):
        for g in range(ngpu):
            torch.cuda.synchronize(g)
        t = time.perf_counter()
        for g, (hi, ho, da, db, s1, s2) in enumerate(res):
            with torch.cuda.device(g):
                with torch.cuda.stream(s1):
                    da.copy_(hi, non_blocking=True)
                with torch.cuda.stream(s2):
                    ho.copy_(db, non_blocking=True)
        for g in range(ngpu):
            torch.cuda.synchronize(g)
        dt = time.perf_counter() - t
        best = dt if best is None else min(best, dt)
    agg = 2 * nbytes * ngpu / best / 1e9
    del res
    return {"gpus": ngpu, "aggregate_bidir_gbs": agg, "per_gpu_bidir_gbs": agg / ngpu}


def kernel_rooflines(torch, S, peaks) -> list:
    """Tenant kernels stand-alone (same device bodies as the dispatcher) on the
    whole GPU; CUDA events on the launching stream; inputs > L2."""
    out = []
    st = torch.cuda.current_stream()

    def time_launch(desc, ins, outs, iters=10, ctas=0):
        S.kernel_launch(0, desc, [a.data_ptr() for a in ins], [a.data_ptr() for a in outs], ctas=ctas,
                        stream=st.cuda_stream)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(iters):
            S.kernel_launch(0, desc, [a.data_ptr() for a in ins], [a.data_ptr() for a in outs], ctas=ctas,
                            stream=st.cuda_stream)
        e1.record(st)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / 1e3 / iters

    n = 1 << 28
    x = torch.empty(n, dtype=torch.float32, device="cuda").uniform_(-1, 1)
    y = torch.empty_like(x)
    for cls, name in ((S.VSCALE, "VSCALE"), (S.XFER, "XFER")):
        t = time_launch(S.make_desc(cls, n=n, alpha=1.001, seed=7), [x], [y])
        gbs = 8 * n / t / 1e9
        out.append({"kernel": name, "bound": "hbm", "size": f"n=2^28 ({8 * n >> 20} MiB moved)",
                    "achieved": round(gbs, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                    "frac": round(gbs / peaks["hbm_gbs"], 4), "ms": round(t * 1e3, 4)})
    del x, y
    # the C2 work item's size on one P=2 partition: what the same body achieves as a
    # stand-alone launch (the ceiling the dispatcher item is judged against)
    n24 = 1 << 24
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    xs = [torch.randint(0, 1 << 30, (n24,), dtype=torch.int32, device="cuda") for _ in range(4)]
    ys = [torch.empty_like(x) for x in xs]         # 4 rotating pairs: 512 MiB > L2
    d24 = S.make_desc(S.XFER, n=n24, seed=7)
    for ctas in ((sms - 4) // 2, sms - 4):          # one KL partition beside the copy partition; two
        for i in range(4):
            S.kernel_launch(0, d24, [xs[i].data_ptr()], [ys[i].data_ptr()], ctas=ctas, stream=st.cuda_stream)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for i in range(20):
            S.kernel_launch(0, d24, [xs[i % 4].data_ptr()], [ys[i % 4].data_ptr()], ctas=ctas,
                            stream=st.cuda_stream)
        e1.record(st)
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1) / 1e3 / 20
        gbs = 8 * n24 / t / 1e9
        out.append({"kernel": "XFER", "bound": "hbm", "size": f"n=2^24 (128 MiB moved) on {ctas} CTAs",
                    "ctas": ctas, "achieved": round(gbs, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                    "frac": round(gbs / peaks["hbm_gbs"], 4), "ms": round(t * 1e3, 4)})
    del xs, ys
    m, nn, k, reps = 128 * 148, 256, 256, 64
    a = torch.randint(-2, 3, (m, k), device="cuda").to(torch.bfloat16)
    b = torch.randint(-2, 3, (k, nn), device="cuda").to(torch.bfloat16)
    c = torch.empty((m, nn), dtype=torch.float32, device="cuda")
    t = time_launch(S.make_desc(S.GEMM, m=m, n=nn, k=k, reps=reps), [a, b], [c], iters=5)
    tf = 2 * m * nn * k * reps / t / 1e12
    out.append({"kernel": "GEMM", "bound": "tensor", "size": f"{m}x{nn}x{k} x R={reps} (148 tiles)",
                "achieved": round(tf, 1), "peak": peaks["bf16_tflops"], "unit": "TFLOP/s",
                "frac": round(tf / peaks["bf16_tflops"], 4), "ms": round(t * 1e3, 4)})
    ref = (a.float() @ b.float())
    assert torch.equal(c, ref), "GEMM roofline run produced a wrong result"
    del a, b, c, ref
    # NEXT-2 tenant kernels (pairwise mix): algorithmic bytes vs the HBM peak
    n = 1 << 30
    xb = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
    hb = torch.zeros(256, dtype=torch.int32, device="cuda")
    t = time_launch(S.make_desc(S.HIST, n=n), [xb], [hb])
    gbs = (n + 1024) / t / 1e9
    out.append({"kernel": "HIST", "bound": "hbm", "size": "n=2^30 bytes -> 256 bins", "achieved": round(gbs, 1),
                "peak": peaks["hbm_gbs"], "unit": "GB/s", "frac": round(gbs / peaks["hbm_gbs"], 4),
                "ms": round(t * 1e3, 4), "note": "shared-memory atomics bound (per-warp sub-histograms)"})
    del xb, hb
    n = 1 << 28
    xs = torch.randint(0, 1 << 20, (n,), dtype=torch.int32, device="cuda")
    ys = torch.empty_like(xs)
    for cls, name, bound in ((S.SCAN, "SCAN", "hbm"), (S.SORT, "SORT", "alu")):
        t = time_launch(S.make_desc(cls, n=n), [xs], [ys])
        gbs = 8 * n / t / 1e9
        out.append({"kernel": name, "bound": bound, "size": "n=2^28 u32" + (", 2048-key segments" if name == "SORT"
                                                                              else ""),
                    "achieved": round(gbs, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                    "frac": round(gbs / peaks["hbm_gbs"], 4), "ms": round(t * 1e3, 4),
                    **({"note": "bitonic network, 66 compare-exchange stages per segment, 2 segments per CTA at once: "
                                "ALU/shuffle bound; "
                                "frac is of the HBM peak, for context"} if name == "SORT" else
                       {"note": "waves scanned from L2 with sums published two waves ahead: the input is read "
                                "from HBM once (8n bytes; 1.05x in ncu)"})})
    del xs, ys
    torch.cuda.empty_cache()
    return out


# ------------------------------------------------------- strings arm
def tstar_device(wl, link, hbm_gbs, tflops, kl_slots: int = 2) -> float:
    """Overlapped roofline T*_d (s) for one physical device running all of wl
    (SURVEY §8(d)): the busiest of the host-link directions (and their
    concurrent sum), HBM, the tensor pipe, the longest per-tenant chain
    (H2D -> KL -> D2H of its jobs back to back, c_t = 1) and, for open-loop
    arrivals, the latest arrival plus its job's chain.  A KL slot owns 1 /
    kl_slots of the SMs (tensor time); HBM is credited at the full peak, so T*
    stays a lower bound."""
    import strings_workload as W
    bh, bd = link["h2d_gbs"] * 1e9, link["d2h_gbs"] * 1e9
    bb = link["bidir_gbs"] * 1e9
    h2d = sum(sum(j.h2d_sizes()) for j in wl.jobs)
    d2h = sum(sum(j.d2h_sizes()) for j in wl.jobs)
    hbm = flop = 0
    chains = {}
    t0 = min(j.arrival_ns for j in wl.jobs) if wl.jobs else 0
    arrival_bound = 0.0
    for j in wl.jobs:
        if j.kclass == W.GEMM:
            jb = 2 * j.m * j.k + 2 * j.k * j.n + 4 * j.m * j.n
            jf = 2 * j.m * j.n * j.k * j.reps
        elif j.kclass == W.HIST:
            jb, jf = j.n + 1024, 0
        else:
            jb, jf = 8 * j.n, 0
        hbm += jb
        flop += jf
        kl = max(jb / (hbm_gbs * 1e9), jf / (tflops * 1e12 / kl_slots))
        one = sum(j.h2d_sizes()) / bh + kl + sum(j.d2h_sizes()) / bd
        chains[j.tenant] = chains.get(j.tenant, 0.0) + one
        arrival_bound = max(arrival_bound, (j.arrival_ns - t0) / 1e9 + one)
    terms = {"h2d": h2d / bh, "d2h": d2h / bd, "bidir": (h2d + d2h) / bb,
             "hbm": (hbm + h2d + d2h) / (hbm_gbs * 1e9), "tensor": flop / (tflops * 1e12),
             "chain": max(chains.values()), "arrival": arrival_bound}
    return max(terms.values()), terms


def run_strings(args, rank, world, torch, gloo):
    import numpy as np

    import strings_workload as W
    from paper_conf_sc_senguptagsp14_b200 import strings as S

    peaks = measured_peaks()
    link = host_link_peaks(torch)
    krl = [] if args.no_kernels else kernel_rooflines(torch, S, peaks)
    torch.cuda.synchronize()

    wl = W.config_c2(jobs_per_tenant=args.jobs_per_tenant)
    for name in ("awake_budget", "admit_cap", "partitions"):
        if getattr(args, name) > 0:
            setattr(wl.config, name, getattr(args, name))
    if args.device_policy >= 0:
        wl.config.device_policy = args.device_policy
    if args.balancer >= 0:
        wl.config.balancer = args.balancer
    cfg = wl.config.resolved()
    # inputs resident in pinned host memory before timing (the H2D phase is part of the job, S4).
    # One input and one output set per tenant, shared by the tenant's jobs: c_t = 1, so a
    # tenant's jobs never overlap, and every job still moves its own bytes each way
    # (1.1 GB of host buffers per rank instead of 8.6 GB; output parity of this configuration
    # with per-job inputs is checked by tests/test_gpu_scheduler.py).
    per_tenant = {}
    for spec in wl.jobs:
        if spec.tenant not in per_tenant:
            per_tenant[spec.tenant] = (
                [torch.from_numpy(a.view(np.uint8).reshape(-1)).pin_memory() for a in W.job_inputs(spec)],
                [torch.empty(sz, dtype=torch.uint8).pin_memory() for sz in spec.d2h_sizes()])
    assert all(t.max_inflight == 1 for t in wl.tenants)
    ins = [per_tenant[spec.tenant][0] for spec in wl.jobs]
    outs = [per_tenant[spec.tenant][1] for spec in wl.jobs]
    arenas = S.torch_arenas(cfg.num_gpus, 1, cfg.admit_cap)      # PyTorch provides the device memory
    S.init_from_config(cfg, timing_mode=S.MEASURED, physical_gpus=1, kl_mode=args.kl_mode,
                       trace_in_memory=bool(args.trace_out), arenas=arenas)
    # the persistent dispatcher now owns every SM: no torch kernels, no device-wide sync until shutdown
    tenants = [S.register_tenant(t.weight, t.max_inflight) for t in wl.tenants]
    stream = torch.cuda.Stream()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def one_step():
        for i, spec in enumerate(wl.jobs):
            S.submit_spec(tenants[spec.tenant], spec, ins[i], outs[i])
        st = S.drain()
        assert st == S.OK, S.strerror(st)

    for _ in range(args.warmup):
        one_step()
    trace_start = len(S.trace()) if args.trace_out else 0
    gloo_barrier(gloo)
    stream.synchronize()
    from paper_conf_sc_senguptagsp14_b200 import parallel as par
    gpu_id = par.physical_gpu(par.rank_info())      # nvidia-smi id of this rank's GPU
    with ClockSampler(gpu_id) as clk:
        ev0.record(stream)
        t_wall = time.perf_counter()
        for _ in range(args.steps):
            one_step()
        ev1.record(stream)
        ev1.synchronize()
        t_wall = time.perf_counter() - t_wall
    gloo_barrier(gloo)
    dt = ev0.elapsed_time(ev1) / 1e3
    trace = S.trace()[trace_start:] if args.trace_out else []
    # steady state: the same K batches submitted back to back, one drain at the end
    # (no per-step pipeline fill/drain; each tenant's jobs still run in order)
    stream.synchronize()
    ev2, ev3 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev2.record(stream)
    for _ in range(args.steps):
        for i, spec in enumerate(wl.jobs):
            S.submit_spec(tenants[spec.tenant], spec, ins[i], outs[i])
    assert S.drain() == S.OK
    ev3.record(stream)
    ev3.synchronize()
    dt_cont = max_over(gloo, ev2.elapsed_time(ev3) / 1e3)
    stats = S.stats()
    infos = [S.job_info(i) for i in range(len(wl.jobs) * (args.warmup + args.steps))]
    jobs_step = len(wl.jobs)
    # e2e: the same workload through the public API from the caller's ordinary
    # (pageable) numpy arrays: the library stages them through its pinned PMT
    # (MOT) and copies results back into the caller's arrays.
    if not args.no_e2e:
        np_t = {t: ([a.numpy().copy() for a in i], [np.empty(o.numel(), dtype=np.uint8) for o in o_])
                for t, (i, o_) in per_tenant.items()}
        np_ins = [np_t[spec.tenant][0] for spec in wl.jobs]
        np_outs = [np_t[spec.tenant][1] for spec in wl.jobs]
        for i, spec in enumerate(wl.jobs):          # warm the staging pool once
            S.submit_spec(tenants[spec.tenant], spec, np_ins[i], np_outs[i])
        assert S.drain() == S.OK
        gloo_barrier(gloo)
        t = time.perf_counter()
        for _ in range(args.steps):
            for i, spec in enumerate(wl.jobs):
                S.submit_spec(tenants[spec.tenant], spec, np_ins[i], np_outs[i])
            assert S.drain() == S.OK
        e2e_dt = time.perf_counter() - t
        e2e = {"value": round(jobs_step * args.steps * world / max_over(gloo, e2e_dt), 3), "unit": "jobs/s",
               "h2d_bytes_per_step": int(sum(sum(j.h2d_sizes()) for j in wl.jobs)),
               "d2h_bytes_per_step": int(sum(sum(j.d2h_sizes()) for j in wl.jobs)),
               "host_buffers": "the caller's own (pageable) numpy arrays: the library stages them into pinned "
                               "memory (PMT/MOT, P:L327-329), DMAs from and to pinned memory, and copies the "
                               "results back into the caller's arrays, all inside the timed region",
               "timer": "wall clock, first strings_submit of a step to strings_drain() return, K steps"}
    else:
        e2e = None
    # the same path with caller-pinned buffers (strings_host_alloc fast path), wall clock
    e2e_pinned = {"value": round(jobs_step * args.steps * world / max_over(gloo, t_wall), 3), "unit": "jobs/s",
                  "host_buffers": "caller-pinned (fast path)",
                  "timer": "wall clock around the K timed steps (value uses CUDA events on the same region)"}
    S.shutdown()
    torch.cuda.synchronize()
    link = max_link(link, host_link_peaks(torch))      # again after the run: the better of both
    # (output parity of this exact configuration is checked by
    # tests/test_gpu_scheduler.py::test_full_size_c2_measured_sampled_parity)
    dt_max = max_over(gloo, dt)
    value = jobs_step * args.steps * world / dt_max
    # per-step spans from the trace -> overlapped roofline fraction
    span_step = dt / args.steps
    tstar, terms = tstar_device(wl, link, peaks["hbm_gbs"], peaks["bf16_tflops_sustained"] or peaks["bf16_tflops"])
    moved = sum(sum(j.h2d_sizes()) + sum(j.d2h_sizes()) for j in wl.jobs)
    link_gbs = moved / span_step / 1e9
    # Jain fairness (Eq. 3, reading R-2) over tenants of the last timed step,
    # secondary form: x_i = (service tenant i received = its busy time on the
    # engines) / (its elapsed time first arrival -> last completion) / w_i
    last = infos[-jobs_step:]
    busy, first, lastd = {}, {}, {}
    for inf in last:
        b = sum(inf.t_done[x] - inf.t_start[x] for x in range(3))
        busy[inf.tenant] = busy.get(inf.tenant, 0) + b
        first[inf.tenant] = min(first.get(inf.tenant, inf.t_arrival), inf.t_arrival)
        lastd[inf.tenant] = max(lastd.get(inf.tenant, 0), inf.t_done[2])
    xs = [busy[t] / max(1, lastd[t] - first[t]) / wl.tenants[t].weight for t in busy]
    from paper_conf_sc_senguptagsp14_b200 import parallel as par_
    jain = par_.jain(par_.gather_over_ranks(gloo, xs))       # over the tenants of all ranks
    # mean completion latency per tenant in the last timed step (all jobs
    # submitted at the start of the step), for the weighted speedup
    step_t0 = min(inf.t_arrival for inf in last)
    mlat = {}
    for inf in last:
        mlat.setdefault(inf.tenant, []).append((inf.t_done[2] - step_t0) / 1e9)
    mlat = {t: sum(v) / len(v) for t, v in mlat.items()}
    # the primary form of R-2: x_i = (T_alone_i / T_shared_i) / w_i, T_alone from
    # each tenant's jobs run alone through the library on this GPU
    alone = alone_mean_latency(S, wl, lambda sp: per_tenant[sp.tenant][0], lambda sp: per_tenant[sp.tenant][1])
    jain_primary, _ = jain_r2(wl, mlat, alone)
    # KL phase: device execution (%globaltimer claim -> last CTA done) vs the
    # host-observed START -> DONE (adds ring pickup + completion notification)
    timed = infos[-jobs_step * args.steps:]
    kl_lat = {}
    for cls, name in ((W.GEMM, "GEMM"), (W.XFER, "XFER")):
        rows = [inf for inf, spec in zip(timed, wl.jobs * args.steps) if spec.kclass == cls]
        dev = sorted((r.kl_gpu_end_ns - r.kl_gpu_start_ns) / 1e3 for r in rows)
        body = sorted((r.kl_gpu_end_ns - r.kl_gpu_exec_ns) / 1e3 for r in rows if r.kl_gpu_exec_ns)
        host = sorted((r.t_done[1] - r.t_start[1]) / 1e3 for r in rows)
        h2d = sorted((r.t_done[0] - r.t_start[0]) / 1e3 for r in rows)
        if dev and name == "XFER":
            # per-op copy rate of the 64 MiB XFER transfers while both directions run
            # (>= 90% of the measured pinned peak; here vs half the bidir peak)
            d2h = sorted((r.t_done[2] - r.t_start[2]) / 1e3 for r in rows)
            nb = 4 * [j for j in wl.jobs if j.kclass == W.XFER][0].n
            kl_lat["XFER_copy_GBps_p50"] = {"h2d": round(nb / max(1e-3, h2d[len(h2d) // 2] * 1e3), 2),
                                            "d2h": round(nb / max(1e-3, d2h[len(d2h) // 2] * 1e3), 2),
                                            "half_bidir_peak": round(link["bidir_gbs"] / 2, 2)}
        if dev:
            kl_lat[name] = {"kl_device_us_p50": round(dev[len(dev) // 2], 1),
                            "kl_device_us_mean": round(sum(dev) / len(dev), 2), "items": len(dev),
                            "kl_body_us_mean": round(sum(body) / len(body), 2) if body else None,
                            "kl_body_us_p50": round(body[len(body) // 2], 1) if body else None,
                            "kl_host_us_p50": round(host[len(host) // 2], 1),
                            "h2d_host_us_p50": round(h2d[len(h2d) // 2], 1)}
    # work items the persistent dispatcher executed in the timed steps: one KL item per
    # job plus the copy partition's items (small H2D/D2H ops), an equal share per step
    kl_items = jobs_step * args.steps + (stats.sm_copy_ops // (args.warmup + 2 * args.steps)) * args.steps
    res = {
        "metric": METRIC, "value": round(value, 3), "unit": "jobs/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt_max / args.steps * 1e3, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16/f32/u32",
        "data": "synthetic (seeded; strings_workload)",
        "config": arm_config(cfg, jobs_step, world, args.kl_mode),
        "continuous": {"value": round(jobs_step * args.steps * world / dt_cont, 3), "unit": "jobs/s",
                       "frac_host_link": round(moved * args.steps / dt_cont / 1e9 / link["bidir_gbs"], 4),
                       "note": "same K batches submitted back to back, one drain (no per-step fill/drain)"},
        # the dominant kernel (the contract's `roofline`): the XFER work item
        "roofline": _kernel_roofline(kl_lat, wl, peaks, krl),
        # the step's dominant resource: the host link
        "roofline_step": {"bound": "host_link", "achieved": round(link_gbs, 2), "peak": round(link["bidir_gbs"], 2),
                          "unit": "GB/s", "frac": round(link_gbs / link["bidir_gbs"], 4), "traffic": None,
                          "resource": "copy engines H2D+D2H (the step's dominant resource)",
                          "peak_source": "measured in this run: concurrent pinned H2D+D2H cudaMemcpyAsync 256 MiB"},
        "overlapped_roofline": {"tstar_ms": round(tstar * 1e3, 3), "span_ms": round(span_step * 1e3, 3),
                                "frac": round(tstar / span_step, 4),
                                "terms_ms": {k: round(v * 1e3, 3) for k, v in terms.items()}},
        "host_link": {k: round(v, 2) for k, v in link.items()},
        "kernel_rooflines": krl,
        "_mean_latency_s_by_tenant": mlat,
        "jain": round(jain_primary, 4),
        "jain_definition": "Eq. (3) over x_i = (T_alone_i / T_shared_i) / w_i (reading R-2): mean completion "
                           "latency of tenant i's jobs in the last timed step vs the same jobs run alone through "
                           "the library on this GPU",
        "jain_service": round(jain, 4),
        "jain_service_definition": "secondary (R-2): x_i = engine-busy service of tenant i / its elapsed time",
        "alone_mean_latency_ms": {W.CLASS_NAMES[k]: round(alone[t] * 1e3, 3) for k, t in
                                  {sp.kclass: sp.tenant for sp in wl.jobs}.items()},
        "phase_latency": kl_lat,
        "gpu_launches": kl_items,
        "gpu_launches_note": "work items executed by the persistent dispatcher kernel (launched once at init): "
                             "KL items plus copy-partition items"
                             if args.kl_mode == 0 else "per-job tenant kernel launches",
        "clocks": clk.summary(),
        "decisions_per_step": (stats.decisions // (args.warmup + 2 * args.steps)),   # warm-up + timed + continuous
        "sm_copy_ops_per_step": (stats.sm_copy_ops // (args.warmup + 2 * args.steps)),
        "sm_copy_note": "H2D/D2H ops of small jobs served by the dispatcher's copy partition (zero-copy SM "
                        "copies over PCIe) instead of the copy engines",
        "decision_us_per_job": round((stats.decision_ns - stats.issue_ns) / 1e3 / max(1, stats.jobs_done), 3),
        "issue_us_per_job": round(stats.issue_ns / 1e3 / max(1, stats.jobs_done), 3),
        "decision_note": "engine-thread time per job: decision core (placement, wake/start passes, epochs, "
                         "feedback) and, separately, issuing its 3 phases' ops (cudaMemcpyAsync, stream "
                         "value writes, KL ring publish)",
        "wall_s": round(t_wall, 4),
    }
    if e2e:
        res["e2e"] = e2e
    res["e2e_pinned"] = e2e_pinned
    if args.trace_out and rank == 0:
        with open(args.trace_out, "w") as f:
            f.write("\n".join(trace) + "\n")
    return res, wl



# ------------------------------------------------ shared measurement helpers
def tenant_buffers(torch, wl):
    """Pinned host buffers, one input and one output set per (tenant, job shape):
    c_t = 1, so a tenant's jobs never overlap, and every job still moves its own
    bytes each way.  Returns (ins_of(spec), outs_of(spec))."""
    import numpy as np

    import strings_workload as W
    bufs = {}
    for spec in wl.jobs:
        key = (spec.tenant, spec.kclass, spec.n, spec.m, spec.k)
        if key not in bufs:
            bufs[key] = ([torch.from_numpy(a.view(np.uint8).reshape(-1)).pin_memory() for a in W.job_inputs(spec)],
                         [torch.empty(sz, dtype=torch.uint8).pin_memory() for sz in spec.d2h_sizes()])
    key = lambda s: (s.tenant, s.kclass, s.n, s.m, s.k)  # noqa: E731
    return (lambda s: bufs[key(s)][0]), (lambda s: bufs[key(s)][1]), bufs


def mean_latency_by_tenant(infos) -> dict:
    """Mean completion latency (s) per tenant of one batch whose jobs were all
    submitted together: JOB_DONE - the batch's first arrival (reading R-1)."""
    t0 = min(i.t_arrival for i in infos)
    lat = {}
    for i in infos:
        lat.setdefault(i.tenant, []).append((i.t_done[2] - t0) / 1e9)
    return {t: sum(v) / len(v) for t, v in lat.items()}


def job_signature(sp) -> tuple:
    return (sp.kclass, sp.n, sp.m, sp.k, sp.reps)


def alone_mean_latency(S, wl, ins_of, outs_of) -> dict:
    """T-bar_alone of reading R-2: each tenant's job sequence run
    ALONE on one GPU through the library (same config, G = 1), its jobs
    submitted together as in the shared run.  Tenants whose job sequences have
    the same shapes (class and sizes, job by job) share one alone run: their
    data differs, which changes no phase's time.  Returns {tenant: mean s}."""
    cfg = dataclasses.replace(wl.config, num_gpus=1, device_weights=None).resolved()
    seqs = {}
    for sp in wl.jobs:
        seqs.setdefault(sp.tenant, []).append(sp)
    groups = {}
    for t, specs in seqs.items():
        groups.setdefault((wl.tenants[t].max_inflight, tuple(job_signature(s) for s in specs)), []).append(t)
    S.init_from_config(cfg, timing_mode=S.MEASURED, physical_gpus=1, trace_in_memory=False)
    out = {}
    try:
        for members in groups.values():
            t = members[0]
            tid = S.register_tenant(wl.tenants[t].weight, wl.tenants[t].max_inflight)
            for _warm in (True, False):
                ids = [S.submit_spec(tid, sp, ins_of(sp), outs_of(sp)) for sp in seqs[t]]
                assert S.drain() == S.OK
            lat = sum(mean_latency_by_tenant([S.job_info(i) for i in ids]).values())
            for m in members:
                out[m] = lat
    finally:
        S.shutdown()
    return out


def jain_r2(wl, shared_lat: dict, alone: dict):
    """Jain's index (Eq. 3) over x_i = (T-bar_alone_i / T-bar_shared_i) / w_i
    (reading R-2, the primary definition: weighted normalised progress)."""
    xs = [alone[t] / shared_lat[t] / wl.tenants[t].weight for t in sorted(shared_lat)]
    return sum(xs) ** 2 / (len(xs) * sum(x * x for x in xs)), xs


def per_gpu_roofline(wl, infos, phys: int, link, peaks, partitions: int, lpg: int) -> list:
    """Overlapped roofline T*_d / span for every physical GPU,
    over the jobs the balancer placed there (logical g -> physical g mod phys)."""
    import strings_workload as W
    by = {}
    for sp, inf in zip(wl.jobs, infos):
        by.setdefault(inf.gid % phys, []).append((sp, inf))
    out = []
    for g in sorted(by):
        rows = by[g]
        sub = W.Workload(f"gpu{g}", wl.config, wl.tenants, [dataclasses.replace(sp, arrival_ns=0) for sp, _ in rows])
        tstar, terms = tstar_device(sub, link, peaks["hbm_gbs"], peaks["bf16_tflops_sustained"] or peaks["bf16_tflops"],
                                    kl_slots=lpg * partitions)
        span = (max(i.t_done[2] for _, i in rows) - min(i.t_start[0] for _, i in rows)) / 1e9
        out.append({"gpu": g, "jobs": len(rows), "tstar_ms": round(tstar * 1e3, 3), "span_ms": round(span * 1e3, 3),
                    "frac": round(tstar / span, 4) if span > 0 else None,
                    "bound_by": max(terms, key=terms.get)})
    return out


def scaled_link(link1: dict, conc: dict) -> dict:
    """Per-GPU link peaks while every GPU copies at once: the alone peaks scaled
    by the concurrent per-GPU bidirectional share (never above the alone peak).
    With one GPU the concurrent test is the alone test again: the better of the
    two measurements is the peak (both are best-of-N timings of the same copies)."""
    if conc["gpus"] == 1:
        b = max(link1["bidir_gbs"], conc["per_gpu_bidir_gbs"])
        return dict(link1, bidir_gbs=b)
    f = min(1.0, conc["per_gpu_bidir_gbs"] / link1["bidir_gbs"])
    return {k: v * f for k, v in link1.items()}


def max_link(a: dict, b: dict) -> dict:
    return {k: max(a[k], b[k]) for k in a}


def run_node(args, torch, gloo, world):
    """N > 1 GPUs in NODE MODE: one process owns all N GPUs and the
    library's level-1 balancer places every job on one of them (the
    runtime overrides the application's GPU choice).  Workload: C2 weak-scaled,
    16 tenants per GPU (16N tenants, 128N jobs per step), DTF joint placement,
    PS dispatch, MEASURED timing.  Beside it, at the same N: static provisioning
    both ways (tenant mod N, and every tenant on device 0), Jain per R-2 from
    alone runs, the overlapped roofline per GPU, and the BASELINE config whose
    G equals N (C1 at 2, C3 at 4, C5 at 8)."""
    import strings_workload as W
    from paper_conf_sc_senguptagsp14_b200 import strings as S

    N = args.gpus
    ngpu = torch.cuda.device_count()
    phys = min(N, ngpu)
    lpg = -(-N // phys)
    peaks = measured_peaks()
    link1 = host_link_peaks(torch)
    conc = host_link_concurrent(torch, phys)
    link = scaled_link(link1, conc)
    wl = W.config_c2(jobs_per_tenant=args.jobs_per_tenant, num_gpus=N)
    for name in ("awake_budget", "admit_cap", "partitions"):
        if getattr(args, name) > 0:
            setattr(wl.config, name, getattr(args, name))
    if args.device_policy >= 0:
        wl.config.device_policy = args.device_policy
    if args.balancer >= 0:
        wl.config.balancer = args.balancer
    cfg = wl.config.resolved()
    ins_of, outs_of, bufs = tenant_buffers(torch, wl)
    arenas = S.torch_arenas(N, phys, cfg.admit_cap)
    torch.cuda.synchronize()
    S.init_from_config(cfg, timing_mode=S.MEASURED, physical_gpus=phys, kl_mode=args.kl_mode,
                       trace_in_memory=False, arenas=arenas)
    tenants = [S.register_tenant(t.weight, t.max_inflight) for t in wl.tenants]
    stream = torch.cuda.Stream(device=0)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ids = []

    def one_step():
        ids.clear()
        for spec in wl.jobs:
            ids.append(S.submit_spec(tenants[spec.tenant], spec, ins_of(spec), outs_of(spec)))
        st = S.drain()
        assert st == S.OK, S.strerror(st)

    for _ in range(args.warmup):
        one_step()
    stream.synchronize()
    timed_ids = []
    with ClockSampler(list(range(phys))) as clk:
        ev0.record(stream)
        t_wall = time.perf_counter()
        for _ in range(args.steps):
            one_step()
            timed_ids.extend(ids)
        ev1.record(stream)
        ev1.synchronize()
        t_wall = time.perf_counter() - t_wall
    dt = max_over(gloo, ev0.elapsed_time(ev1) / 1e3)
    infos = [S.job_info(i) for i in ids]            # the last timed step
    # the dominant kernel: XFER work items of every timed step on every GPU (device stamps)
    xf = [S.job_info(i) for i, sp in zip(timed_ids, wl.jobs * args.steps) if sp.kclass == W.XFER]
    dev_us = sorted((r.kl_gpu_end_ns - r.kl_gpu_start_ns) / 1e3 for r in xf if r.kl_gpu_end_ns)
    body_us = sorted((r.kl_gpu_end_ns - r.kl_gpu_exec_ns) / 1e3 for r in xf if r.kl_gpu_exec_ns)
    kl_lat = {}
    if dev_us:
        kl_lat["XFER"] = {"kl_device_us_p50": round(dev_us[len(dev_us) // 2], 1),
                          "kl_device_us_mean": round(sum(dev_us) / len(dev_us), 2), "items": len(dev_us),
                          "kl_body_us_mean": round(sum(body_us) / len(body_us), 2) if body_us else None,
                          "kl_body_us_p50": round(body_us[len(body_us) // 2], 1) if body_us else None}
    stats = S.stats()
    jobs_step = len(wl.jobs)
    e2e = None
    if not args.no_e2e:
        import numpy as np
        np_bufs = {k: ([a.numpy().copy() for a in i], [np.empty(o.numel(), dtype=np.uint8) for o in o_])
                   for k, (i, o_) in bufs.items()}
        key = lambda s: (s.tenant, s.kclass, s.n, s.m, s.k)  # noqa: E731
        for spec in wl.jobs:                         # warm the staging pool once
            S.submit_spec(tenants[spec.tenant], spec, np_bufs[key(spec)][0], np_bufs[key(spec)][1])
        assert S.drain() == S.OK
        e2e_steps = max(1, min(args.steps, 5))
        t = time.perf_counter()
        for _ in range(e2e_steps):
            for spec in wl.jobs:
                S.submit_spec(tenants[spec.tenant], spec, np_bufs[key(spec)][0], np_bufs[key(spec)][1])
            assert S.drain() == S.OK
        e2e_dt = time.perf_counter() - t
        e2e = {"value": round(jobs_step * e2e_steps / e2e_dt, 3), "unit": "jobs/s", "steps": e2e_steps,
               "h2d_bytes_per_step": int(sum(sum(j.h2d_sizes()) for j in wl.jobs)),
               "d2h_bytes_per_step": int(sum(sum(j.d2h_sizes()) for j in wl.jobs)),
               "host_buffers": "the caller's own (pageable) numpy arrays, staged by the library (PMT/MOT, "
                               "P:L327-329) inside the timed region",
               "timer": "wall clock, first strings_submit to strings_drain() return"}
        del np_bufs
    S.shutdown()
    del arenas
    torch.cuda.synchronize()
    # the link peaks again after the run (best of both: a peak must not be an underestimate)
    link1 = max_link(link1, host_link_peaks(torch))
    c2 = host_link_concurrent(torch, phys)
    if c2["aggregate_bidir_gbs"] > conc["aggregate_bidir_gbs"]:
        conc = c2
    link = scaled_link(link1, conc)
    value = jobs_step * args.steps / dt
    moved = sum(sum(j.h2d_sizes()) + sum(j.d2h_sizes()) for j in wl.jobs)
    span_step = dt / args.steps
    link_gbs = moved / span_step / 1e9
    agg_peak = link["bidir_gbs"] * phys
    shared = mean_latency_by_tenant(infos)
    alone = alone_mean_latency(S, wl, ins_of, outs_of)
    jain, xs = jain_r2(wl, shared, alone)
    per_gpu = per_gpu_roofline(wl, infos, phys, link, peaks, cfg.partitions, lpg)
    placed = {}
    for inf in infos:
        placed[inf.gid] = placed.get(inf.gid, 0) + 1
    res = {
        "metric": METRIC, "value": round(value, 3), "unit": "jobs/s", "n_gpus": N,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt / args.steps * 1e3, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16/f32/u32",
        "data": "synthetic (seeded; strings_workload)",
        "config": {"workload": f"C2 weak-scaled to {N} GPUs: {len(wl.tenants)} tenants (GEMM 256^3 R=64 / XFER "
                               f"2^24 u32 alternating) x {args.jobs_per_tenant} jobs, DTF joint placement over "
                               f"{N} devices, PS dispatch, measured timing",
                   "jobs_per_step": jobs_step, "partitions": cfg.partitions, "awake_budget": cfg.awake_budget,
                   "admit_cap": cfg.admit_cap, "l2": "inputs larger than L2 (4 GiB each way per GPU per step)",
                   "parallelism": f"node mode, {W.BALANCER_NAMES[cfg.balancer]} balancer: one process places "
                                  f"every job on one of {N} devices ({phys} physical GPU(s))"
                                  + ("" if phys == N else "; LOGICAL devices share GPUs: not an N-GPU number"),
                   "ranks": f"{world} (rank 0 drives the node; other ranks idle: no data-path collective)",
                   "kl_mode": "persistent dispatcher" if stats.kl_mode == 0 else "per-op launches"},
        "placement": {str(g): placed.get(g, 0) for g in range(N)},
        # the dominant kernel (the contract's `roofline`): the XFER work items on every GPU
        "roofline": _kernel_roofline(kl_lat, wl, peaks),
        "roofline_step": {"bound": "host_link", "achieved": round(link_gbs, 2), "peak": round(agg_peak, 2),
                     "unit": "GB/s", "frac": round(link_gbs / agg_peak, 4), "traffic": None,
                     "resource": f"copy engines H2D+D2H of {phys} GPU(s)",
                     "peak_source": "measured in this run: pinned H2D+D2H 256 MiB copies on every GPU at once"},
        "per_gpu_roofline": per_gpu,
        "per_gpu_roofline_min": min((d["frac"] for d in per_gpu if d["frac"]), default=None),
        "host_link": {"alone": {k: round(v, 2) for k, v in link1.items()},
                      "concurrent": {k: round(v, 2) if isinstance(v, float) else v for k, v in conc.items()}},
        "jain": round(jain, 4),
        "jain_definition": "Eq. (3) over x_i = (T_alone_i / T_shared_i) / w_i (reading R-2): mean completion "
                           "latency of tenant i's jobs in the last timed step vs the same class's jobs run alone "
                           "through the library on one GPU",
        "alone_mean_latency_ms": {W.CLASS_NAMES[k]: round(alone[t] * 1e3, 3) for k, t in
                                  {sp.kclass: sp.tenant for sp in wl.jobs}.items()},
        "gpu_launches": jobs_step * args.steps if stats.kl_mode == 0 else jobs_step * args.steps,
        "gpu_launches_note": "KL work items executed by the persistent dispatcher kernels (one launch per GPU at "
                             "init), one per job; plus copy-partition items" if stats.kl_mode == 0 else
                             "per-job tenant kernel launches",
        "clocks": clk.summary(),
        "decision_us_per_job": round((stats.decision_ns - stats.issue_ns) / 1e3 / max(1, stats.jobs_done), 3),
        "issue_us_per_job": round(stats.issue_ns / 1e3 / max(1, stats.jobs_done), 3),
        "wall_s": round(t_wall, 4),
    }
    if e2e:
        res["e2e"] = e2e
    if not args.no_static:
        from paper_conf_sc_senguptagsp14_b200.static_baseline import run_static
        reps = max(5, args.static_repeats)
        sb = {"tenant_mod_N": run_static(wl, num_gpus=phys, policy="mod", repeats=reps),
              "device_0": run_static(wl, num_gpus=phys, policy="zero", repeats=reps)}
        for k in sb:
            lat = sb[k].pop("mean_latency_s_by_tenant")
            sb[k]["weighted_speedup_strings"] = round(sum(lat[t] / shared[t] for t in shared) / len(shared), 3)
        res["static_baseline"] = sb
        res["speedup_vs_static"] = round(value / sb["tenant_mod_N"]["value"], 3)
        res["speedup_vs_static_device0"] = round(value / sb["device_0"]["value"], 3)
        res["weighted_speedup_vs_static"] = sb["tenant_mod_N"]["weighted_speedup_strings"]
    if not args.no_baseline_config:
        name = {2: "C1", 4: "C3", 8: "C5"}.get(N)
        if name:
            # (its own static baselines only on request: at N = 8 they spawn 2 x 128 processes)
            res["baseline_config"] = config_result(torch, name, phys, link, peaks, repeats=2, warmups=1,
                                                   static=args.baseline_config_static and not args.no_static)
    return res, wl


def arm_config(cfg, jobs_step: int, world: int, kl_mode: int) -> dict:
    """The `config` object of the JSON line (both arms print the same one)."""
    return {"workload": "C2: 16 tenants (8 GEMM 256^3 R=64, 8 XFER 2^24 u32) x 8 jobs, 1 B200 per rank, "
                        "DTF joint placement, PS dispatch, measured timing",
            "jobs_per_step_per_gpu": jobs_step, "partitions": cfg.partitions,
            "awake_budget": cfg.awake_budget, "admit_cap": cfg.admit_cap,
            "l2": "inputs larger than L2 (4 GiB H2D + 4 GiB D2H per step)",
            "kl_mode": "persistent dispatcher" if kl_mode == 0 else "per-job launches",
            "parallelism": f"placement only, {world} rank(s) x 1 GPU" + (
                " (TEST MODE: all ranks share one GPU, SM-limited dispatchers; not a reported number)"
                if os.environ.get("STRINGS_BENCH_SHARE_GPU") == "1" else "")}


def _kernel_roofline(kl_lat, wl, peaks, krl=None) -> dict:
    """The dominant kernel work inside the timed step: XFER items run by the
    persistent dispatcher on one P=2 SM partition (72 SMs beside the 4-CTA copy
    partition, plus the sibling slot's 72 when it is idle), HBM-bound.
    achieved = algorithmic bytes per item (read + write) / MEAN device
    time of the timed region's items (%globaltimer: leader claim -> last CTA
    done; a launch of the persistent kernel is one work item, and CUDA events
    cannot bracket an item inside a resident kernel).  Beside it: the median,
    the body alone, the same body launched stand-alone on the same CTA count
    (measured in this run, kernel_rooflines) and the ncu DRAM traffic of that
    launch."""
    import strings_workload as W
    x = kl_lat.get("XFER")
    n = [j for j in wl.jobs if j.kclass == W.XFER][0].n
    if not x or not x["kl_device_us_p50"]:
        return None                                  # kl_mode 1: no dispatcher stamps
    gbs = 8 * n / (x["kl_device_us_mean"] * 1e3)
    gbs50 = 8 * n / (x["kl_device_us_p50"] * 1e3)
    out = {"kernel": "dispatcher XFER item (fmix32, TMA bulk pipeline, dynamic chunk claiming)", "bound": "hbm",
           "achieved": round(gbs, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
           "frac": round(gbs / peaks["hbm_gbs"], 4), "traffic": _XFER_ITEM_NCU["dram_bytes"],
           "traffic_source": _XFER_ITEM_NCU["source"], "items_timed": x["items"],
           "duration_us_mean": x["kl_device_us_mean"], "duration_us_p50": x["kl_device_us_p50"],
           "frac_p50": round(gbs50 / peaks["hbm_gbs"], 4),
           "peak_source": peaks["source"] + " hbm_gbs",
           "bytes_per_launch": 8 * n, "note": "per work item on its KL slot's 72 SMs plus the sibling slot's 72 "
           "when that one is idle (lent CTAs, STRINGS_KL_HELP); otherwise the other slot runs its own item and "
           "shares HBM; device time includes the claim, broadcast and completion publish (stand-alone full-GPU "
           "runs: kernel_rooflines)"}
    if x.get("kl_body_us_mean"):
        # the body alone (leader's body start -> last CTA done): without the claim and
        # the partition broadcast, which are dispatch cost, not kernel work
        bg = 8 * n / (x["kl_body_us_mean"] * 1e3)
        out["body_only"] = {"achieved": round(bg, 1), "frac": round(bg / peaks["hbm_gbs"], 4),
                            "us_mean": x["kl_body_us_mean"], "us_p50": x["kl_body_us_p50"]}
    same = sorted((k for k in (krl or []) if k.get("ctas") and k["kernel"] == "XFER"), key=lambda k: k["ctas"])
    if same:
        out["same_work_standalone"] = {"ctas": same[0]["ctas"], "GBps": same[0]["achieved"],
                                       "us": round(same[0]["ms"] * 1e3, 2),
                                       "item_vs_standalone": round(gbs / same[0]["achieved"], 4)}
    return out


# ncu --set full of the C2 work item's body as a stand-alone launch (XFER 2^24 u32
# on 144 CTAs -- one KL partition plus its lent sibling -- `tools/kernel_probe.py
# xfer_item`): dram__bytes_read.sum + dram__bytes_write.sum per launch, mean of two
# launches; profiles/r02_kernels.md.  Reads 67.14 MB = the 64 MiB input exactly;
# writes 17.3 MB of 67.1 MB: most of the output is still in the 126 MB L2 when the
# launch ends (no re-reads).
_XFER_ITEM_NCU = {"dram_bytes": 67136768 + 17278080,
                  "source": "profiles/r02_kernels.md (xfer_item: ncu --set full, XFER 2^24 on 144 CTAs)"}


def max_over(gloo, x: float) -> float:
    from paper_conf_sc_senguptagsp14_b200 import parallel as par
    return par.max_over_ranks(gloo, x)


def gloo_barrier(gloo):
    from paper_conf_sc_senguptagsp14_b200 import parallel as par
    par.barrier(gloo)


# --------------------------------------------------------------- baselines
def _oracle_inputs(specs):
    import numpy as np

    import strings_workload as W
    ins = [W.job_inputs(s) for s in specs]
    outs = [[np.empty(sh, dt) for sh, dt in W.job_output_shapes(s)] for s in specs]
    return ins, outs


def cpu_baseline(wl, threads: int = 0) -> dict:
    """SURVEY §8(d)'s CPU reference: the oracle's plain C kernels (oracle/c,
    -O3, no BLAS), the WHOLE workload -- every job's H2D bytes copied in, the
    kernel (GEMM repeated R times), the D2H bytes copied out -- on a pthread pool
    of `threads` workers (default: every host core), tenants dealt round-robin
    to workers and each tenant's jobs run in submission order (c_t = 1).
    Inputs are generated before timing.  Also the DES speed: the oracle's
    discrete-event model of the scheduler (plain Python) over the workload."""
    from oracle import cbind
    from oracle.des import run_oracle

    threads = threads or (os.cpu_count() or 1)
    ins, outs = _oracle_inputs(wl.jobs)
    cbind.lib()
    t = time.perf_counter()
    cbind.run_jobs(wl.jobs, ins, outs, threads)
    dt = time.perf_counter() - t
    # one core (SURVEY §8(d) asks for both): one job of each class of the workload
    # in submission order, on one worker
    firsts = {}
    for i, spec in enumerate(wl.jobs):
        firsts.setdefault(spec.kclass, i)
    pick = sorted(firsts.values())
    t1 = time.perf_counter()
    cbind.run_jobs([wl.jobs[i] for i in pick], [ins[i] for i in pick], [outs[i] for i in pick], 1)
    dt1 = time.perf_counter() - t1
    t2 = time.perf_counter()
    o = run_oracle(wl)
    des = time.perf_counter() - t2
    decisions = sum(1 for ln in o.trace if " PLACE " in ln or " WAKE " in ln)
    busy = min(threads, len({s.tenant for s in wl.jobs}))
    return {"value": round(len(wl.jobs) / dt, 3), "unit": "jobs/s", "cores": busy, "kind": "oracle",
            "sample": f"the whole workload ({len(wl.jobs)} jobs, GEMM R = {max(s.reps for s in wl.jobs)} computed "
                      f"every repetition) through the oracle's plain C kernels (oracle/c/kernels.c, gcc -O3, no "
                      f"BLAS) with host copies in and out, {threads} worker threads ({busy} busy: tenants are "
                      f"dealt to workers, c_t = 1)",
            "seconds": round(dt, 3),
            "one_core": {"value": round(len(pick) / dt1, 3), "unit": "jobs/s", "cores": 1,
                         "sample": f"{len(pick)} jobs, the first of each class in the workload, one worker",
                         "seconds": round(dt1, 3)},
            "des": {"seconds": round(des, 3), "decisions": decisions,
                    "decisions_per_s": round(decisions / des, 1) if des > 0 else None,
                    "note": "oracle/des.py (plain Python) on the same workload"}}


def run_reference(args):
    """--impl reference: the oracle as it stands on the host cores, same
    config/metric.  Each step is a bounded sample of C2: one job per tenant (16
    jobs, GEMM R = 64 computed every repetition) through the oracle's plain C
    kernels on a pool of every host core, host copies in and out."""
    import strings_workload as W
    from oracle import cbind

    wl = W.config_c2(jobs_per_tenant=args.jobs_per_tenant)
    sample = [s for s in wl.jobs if s.arrival_ns == 0][:len(wl.tenants)]
    ins, outs = _oracle_inputs(sample)
    threads = os.cpu_count() or 1
    cbind.lib()
    for _ in range(args.warmup):
        cbind.run_jobs(sample[:2], ins[:2], outs[:2], threads)
    t = time.perf_counter()
    for _ in range(args.steps):
        cbind.run_jobs(sample, ins, outs, threads)
    dt = time.perf_counter() - t
    v = round(len(sample) * args.steps / dt, 3)
    busy = min(threads, len(sample))
    line = {"metric": METRIC, "value": v, "unit": "jobs/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(dt / args.steps * 1e3, 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64/f32/u32 (plain C)", "data": "synthetic",
            "impl": "reference",
            "config": arm_config(wl.config.resolved(), len(wl.jobs), args.gpus, args.kl_mode),
            "reference_note": "the oracle (oracle/c/kernels.c, plain C, -O3, no BLAS) runs the C2 jobs on the host: "
                              "copy-in, CPU kernel (GEMM R = 64 times), copy-out; each step is one job per tenant",
            "cpu_baseline": {"value": v, "unit": "jobs/s", "cores": busy, "kind": "oracle",
                             "sample": f"16 jobs of C2 per step (one per tenant) on {threads} threads"},
            "e2e": {"value": v, "unit": "jobs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def policy_sweep(args) -> None:
    """Paper-style policy comparison (Figs 12-15 analogue) on C2, one B200."""
    import numpy as np
    import torch

    import strings_workload as W
    from paper_conf_sc_senguptagsp14_b200 import strings as S
    from paper_conf_sc_senguptagsp14_b200.static_baseline import run_static

    base = W.config_c2(jobs_per_tenant=args.jobs_per_tenant)
    ins = [[torch.from_numpy(a.view(np.uint8).reshape(-1)).pin_memory() for a in W.job_inputs(sp)]
           for sp in base.jobs]
    outs = [[torch.empty(sz, dtype=torch.uint8).pin_memory() for sz in sp.d2h_sizes()] for sp in base.jobs]
    st = run_static(base, num_gpus=1, repeats=3)
    static_lat = st["mean_latency_s_by_tenant"]
    rows = []
    combos = [(W.DTF, d) for d in (W.FIFO, W.LAS, W.PS, W.TFS)] + \
             [(b, W.PS) for b in (W.GRR, W.GMIN, W.RTF, W.GUF, W.MBF, W.DYNAMIC)]
    for bal, dev in combos:
        cfg = W.config_c2(jobs_per_tenant=args.jobs_per_tenant).config
        cfg.balancer, cfg.device_policy = bal, dev
        cfg = cfg.resolved()
        S.init_from_config(cfg, timing_mode=S.MEASURED, physical_gpus=1)
        tenants = [S.register_tenant(t.weight, t.max_inflight) for t in base.tenants]
        spans, lat = [], {}
        for step in range(2 + args.steps):
            t0 = time.perf_counter()
            first = None
            for i, sp in enumerate(base.jobs):
                jid = S.submit_spec(tenants[sp.tenant], sp, ins[i], outs[i])
                first = jid if first is None else first
            assert S.drain() == S.OK
            if step >= 2:
                spans.append(time.perf_counter() - t0)
                infos = [S.job_info(first + i) for i in range(len(base.jobs))]
                t_arr = min(x.t_arrival for x in infos)
                for x in infos:
                    lat.setdefault(x.tenant, []).append((x.t_done[2] - t_arr) / 1e9)
        S.shutdown()
        mlat = {t: sum(v) / len(v) for t, v in lat.items()}
        ws = sum(static_lat[t] / mlat[t] for t in mlat) / len(mlat)
        xs = [1.0 / mlat[t] for t in mlat]          # progress rate per tenant (equal weights)
        jain = sum(xs) ** 2 / (len(xs) * sum(x * x for x in xs))
        rows.append({"balancer": W.BALANCER_NAMES[bal], "device_policy": W.DEVICE_POLICY_NAMES[dev],
                     "jobs_per_s": round(len(base.jobs) / statistics.median(spans), 1),
                     "weighted_speedup_vs_static": round(ws, 3), "jain_progress": round(jain, 4)})
        print(json.dumps(rows[-1]), flush=True)
    print(json.dumps({"sweep": "C2 on 1 B200", "static_jobs_per_s": round(st["value"], 1), "rows": rows}))


def fig2(args) -> None:
    """PAPER.md L67-73 (Fig. 2): identical MonteCarlo-like requests issued one
    after another vs co-resident on streams of one context.  Here: 8 identical
    transfer-heavy XFER jobs (64 MiB each way) (a) from one tenant, strictly
    sequential; (b) from 8 tenants co-scheduled by Strings (PS); (c) from 8
    separate processes/contexts (static provisioning)."""
    import numpy as np
    import torch

    import strings_workload as W
    from paper_conf_sc_senguptagsp14_b200 import strings as S
    from paper_conf_sc_senguptagsp14_b200.static_baseline import run_static

    n_req = 8
    specs = [W.with_nominal_durations(W._xfer(t, 100 + t)) for t in range(n_req)]
    ins = [[torch.from_numpy(a.view(np.uint8).reshape(-1)).pin_memory() for a in W.job_inputs(sp)] for sp in specs]
    outs = [[torch.empty(sz, dtype=torch.uint8).pin_memory() for sz in sp.d2h_sizes()] for sp in specs]
    res = {"requests": n_req, "request": "XFER n=2^24 (64 MiB H2D + 64 MiB D2H)"}
    for name, tenants_n in (("sequential_one_tenant", 1), ("coresident_strings_ps", n_req)):
        S.init(num_gpus=1, physical_gpus=1, balancer=W.GMIN, device_policy=W.PS, timing_mode=S.MEASURED)
        ts = [S.register_tenant(1, 1) for _ in range(tenants_n)]
        spans = []
        for rep in range(2 + args.steps):
            t0 = time.perf_counter()
            for i, sp in enumerate(specs):
                S.submit(ts[i % tenants_n], S.make_desc(S.XFER, n=sp.n, seed=sp.seed), ins[i], outs[i])
            assert S.drain() == S.OK
            if rep >= 2:
                spans.append(time.perf_counter() - t0)
        S.shutdown()
        res[name + "_ms"] = round(statistics.median(spans) * 1e3, 3)
    wl = W.Workload("fig2", W.SystemConfig(num_gpus=1), [W.TenantSpec() for _ in range(n_req)],
                    [W.JobSpec(**vars(sp)) for sp in specs])
    st = run_static(wl, num_gpus=1, repeats=3)
    res["separate_contexts_static_ms"] = round(st["span_s"] * 1e3, 3)
    res["coresident_vs_sequential"] = round(res["sequential_one_tenant_ms"] / res["coresident_strings_ps_ms"], 3)
    res["coresident_vs_separate_contexts"] = round(res["separate_contexts_static_ms"] / res["coresident_strings_ps_ms"], 3)
    print(json.dumps(res))


def copy_replay_s(torch, wl, streams_per_dir: int, reps: int = 2) -> float:
    """Physical floor of a config's host-link traffic: every job's H2D and D2H
    buffers copied with plain cudaMemcpyAsync (pinned host memory), jobs dealt
    round-robin over `streams_per_dir` streams per direction, no kernels, no
    dependencies, no scheduling.  Every stream is first held by a spin kernel
    while all copies are queued behind it, so host issue cost is excluded; the
    time is taken with CUDA events from the first stream's release to the last
    stream's end.  Best of `reps`."""
    h2d = [b for j in wl.jobs for b in j.h2d_sizes() if b]
    d2h = [b for j in wl.jobs for b in j.d2h_sizes() if b]
    big = max(h2d + d2h + [1])
    hsrc = torch.empty(big, dtype=torch.uint8).pin_memory()
    hdst = torch.empty(big, dtype=torch.uint8).pin_memory()
    dsrc = torch.empty(big, dtype=torch.uint8, device="cuda")
    ddst = torch.empty(big, dtype=torch.uint8, device="cuda")
    streams = [torch.cuda.Stream() for _ in range(2 * streams_per_dir)]
    sh, sd = streams[:streams_per_dir], streams[streams_per_dir:]
    hold = int(2e9 * max(0.05, 60e-6 * (len(h2d) + len(d2h))))      # cycles: outlast the issue loop
    best = None
    for _ in range(reps):
        torch.cuda.synchronize()
        t0, t1 = [], []
        for st in streams:
            with torch.cuda.stream(st):
                torch.cuda._sleep(hold)
                e = torch.cuda.Event(enable_timing=True)
                e.record(st)
                t0.append(e)
        for i in range(max(len(h2d), len(d2h))):
            if i < len(h2d):
                with torch.cuda.stream(sh[i % streams_per_dir]):
                    ddst[:h2d[i]].copy_(hsrc[:h2d[i]], non_blocking=True)
            if i < len(d2h):
                with torch.cuda.stream(sd[i % streams_per_dir]):
                    hdst[:d2h[i]].copy_(dsrc[:d2h[i]], non_blocking=True)
        for st in streams:
            e = torch.cuda.Event(enable_timing=True)
            e.record(st)
            t1.append(e)
        torch.cuda.synchronize()
        ref = t0[0]
        first = min(ref.elapsed_time(e) for e in t0)
        last = max(ref.elapsed_time(e) for e in t1)
        dt = (last - first) / 1e3
        best = dt if best is None else min(best, dt)
    del hsrc, hdst, dsrc, ddst
    return best


def config_result(torch, name: str, ngpu: int, link, peaks, repeats: int = 5, static: bool = False,
                  replay: bool = False, seed: int = 1, warmups: int = 2) -> dict:
    """One BASELINE configuration at full size, MEASURED timing, node mode (one
    process, G logical devices mapped round-robin onto `ngpu` GPUs), workload
    seed `seed`.  `warmups` untimed runs, then `repeats` timed runs (SURVEY
    §8(d): 2 warm-up, 5 timed per seed); the median jobs/s and span,
    the overlapped roofline T*/span per physical GPU over the jobs placed there
    (SURVEY §8(d)), Jain per R-2 (alone runs), optionally static provisioning
    (tenant mod GPUs, and device 0) and the plain-copy replay."""
    import strings_workload as W
    from paper_conf_sc_senguptagsp14_b200 import strings as S

    wl = W.CONFIGS[name](seed=seed)
    if os.environ.get("BENCH_AWAKE_BUDGET"):       # experiments: override A (M follows unless set)
        wl.config.awake_budget = int(os.environ["BENCH_AWAKE_BUDGET"])
    if os.environ.get("BENCH_ADMIT_CAP"):
        wl.config.admit_cap = int(os.environ["BENCH_ADMIT_CAP"])
    # arrivals are submit times in MEASURED mode: the whole config is offered at t = 0
    wl = dataclasses.replace(wl, jobs=[dataclasses.replace(j, arrival_ns=0) for j in wl.jobs])
    cfg = wl.config.resolved()
    lpg = max(1, -(-cfg.num_gpus // ngpu))       # logical devices per GPU
    ins_of, outs_of, bufs = tenant_buffers(torch, wl)
    runs = []
    for rep in range(warmups + repeats):
        S.init_from_config(cfg, timing_mode=S.MEASURED, physical_gpus=ngpu, trace_in_memory=False)
        ts = [S.register_tenant(t.weight, t.max_inflight) for t in wl.tenants]
        t0 = time.perf_counter()
        ids = [S.submit_spec(ts[sp.tenant], sp, ins_of(sp), outs_of(sp)) for sp in wl.jobs]
        st = S.drain()
        wall = time.perf_counter() - t0
        infos = [S.job_info(i) for i in ids]
        stats = S.stats()
        S.shutdown()
        if rep < warmups:
            continue                    # warm-up
        span = (max(i.t_done[2] for i in infos) - min(i.t_arrival for i in infos)) / 1e9
        runs.append({"span": span, "wall": wall, "status": st, "infos": infos, "sm_copy_ops": stats.sm_copy_ops,
                     "failed": sum(1 for i in infos if i.status != S.OK),
                     "decision_us": (stats.decision_ns - stats.issue_ns) / 1e3 / max(1, stats.jobs_done),
                     "issue_us": stats.issue_ns / 1e3 / max(1, stats.jobs_done)})
    runs.sort(key=lambda r: r["span"])
    mid = runs[len(runs) // 2]
    span = mid["span"]
    tstar, terms = tstar_device(wl, link, peaks["hbm_gbs"], peaks["bf16_tflops_sustained"] or peaks["bf16_tflops"],
                                kl_slots=lpg * cfg.partitions)
    per_gpu = per_gpu_roofline(wl, mid["infos"], ngpu, link, peaks, cfg.partitions, lpg)
    shared = mean_latency_by_tenant(mid["infos"])
    alone = alone_mean_latency(S, wl, ins_of, outs_of)
    jain, _ = jain_r2(wl, shared, alone)
    out = {"config": name, "seed": seed, "jobs": len(wl.jobs), "tenants": len(wl.tenants),
           "logical_gpus": cfg.num_gpus, "physical_gpus": ngpu,
           "balancer": W.BALANCER_NAMES[cfg.balancer], "las_admission": cfg.las_admission,
           "device_policy": W.DEVICE_POLICY_NAMES[cfg.device_policy],
           "status": max((r["status"] for r in runs), key=abs),
           "failed_jobs": sum(r["failed"] for r in runs),
           "jobs_per_s": round(len(wl.jobs) / span, 1),
           "span_ms": round(span * 1e3, 2), "span_ms_min_max": [round(runs[0]["span"] * 1e3, 2),
                                                             round(runs[-1]["span"] * 1e3, 2)],
           "runs": len(runs), "warmup_runs": warmups, "sm_copy_ops": mid["sm_copy_ops"],
           "tstar_ms": round(tstar * 1e3, 3) if ngpu == 1 else None,
           "roofline_frac": round(tstar / span, 4) if ngpu == 1 else None,
           "tstar_terms_ms": {k: round(v * 1e3, 3) for k, v in terms.items()} if ngpu == 1 else None,
           "per_gpu_roofline": per_gpu,
           "per_gpu_roofline_min": min((d["frac"] for d in per_gpu if d["frac"]), default=None),
           "jain": round(jain, 4), "jain_definition": "R-2: x_i = (T_alone_i / T_shared_i) / w_i",
           "decision_us_per_job": round(mid["decision_us"], 3), "issue_us_per_job": round(mid["issue_us"], 3),
           "host_link_gbs": {k: round(v, 2) for k, v in link.items()},
           "note": "logical devices share the physical GPUs' host links and SMs"
           if cfg.num_gpus > ngpu else "one logical device per GPU"}
    if replay:
        rp = copy_replay_s(torch, wl, lpg)
        out["copy_replay_ms"] = round(rp * 1e3, 3)
        out["frac_vs_copy_replay"] = round(rp / span, 4)
        out["copy_replay_note"] = ("the config's H2D + D2H buffers copied with plain cudaMemcpyAsync, "
                                   f"{lpg} stream(s) per direction (jobs dealt round-robin), all pre-queued, no "
                                   "kernels or dependencies: what plain copies of these sizes achieve")
    if static:
        from paper_conf_sc_senguptagsp14_b200.static_baseline import run_static
        for pol, key in (("mod", "static_tenant_mod_gpus"), ("zero", "static_device_0")):
            sb = run_static(wl, num_gpus=ngpu, policy=pol, repeats=repeats)
            lat = sb.pop("mean_latency_s_by_tenant")
            sb["weighted_speedup_strings"] = round(sum(lat[t] / shared[t] for t in shared) / len(shared), 3)
            out[key] = sb
            out["speedup_vs_" + key] = round(out["jobs_per_s"] / sb["value"], 3)
    del bufs
    return out


def run_configs(args) -> None:
    """All five BASELINE.json configurations at full size (config_result), one
    JSON line each.  BENCH_CONFIGS selects a subset; --config-static adds the
    static baselines."""
    import torch

    ngpu = torch.cuda.device_count()
    peaks = measured_peaks()
    link1 = host_link_peaks(torch)
    link = scaled_link(link1, host_link_concurrent(torch, ngpu)) if ngpu > 1 else link1
    for name in os.environ.get("BENCH_CONFIGS", "C1,C2,C3,C4,C5").split(","):
        for seed in (int(x) for x in args.config_seeds.split(",")):
            print(json.dumps(config_result(torch, name, ngpu, link, peaks, repeats=args.config_repeats,
                                           static=args.config_static, replay=True, seed=seed)), flush=True)


def _pct(xs, q):
    xs = sorted(xs)
    return xs[min(len(xs) - 1, int(q * len(xs)))] if xs else None


def open_loop(args) -> None:
    """C4 as the open-loop system SURVEY §8(d) describes: 64 tenants whose jobs
    arrive by Eq. (4) at offered load rho = 0.9 per device, skewed
    priorities w = 8/4/2/1.  A submitter thread of this process calls
    strings_submit at each job's arrival time (MEASURED timing, caller-pinned
    buffers), so a job's latency is done - submit on the library clock.  On a box
    with fewer GPUs than the config's 8 devices the arrival times are dilated by
    the number of logical devices per GPU, which keeps the offered load per
    physical host link at rho.  Two schedulers see the same arrivals:
    the config's (weighted-LAS admission + GUF placement, LAS wake order) and an
    arrival-order baseline (GMin placement, FIFO wake order).  Reported per
    priority class: jobs, p50 / p99 / mean latency; plus jobs/s (bounded by the
    arrival rate), T*/span with T* including the arrival-bound term, Jain, and
    the submitter's lateness."""
    import threading

    import torch

    import strings_workload as W
    from paper_conf_sc_senguptagsp14_b200 import strings as S

    ngpu = torch.cuda.device_count()
    peaks = measured_peaks()
    link = host_link_peaks(torch)
    base = W.CONFIGS[args.open_loop_config]()
    lpg = max(1, (base.config.num_gpus + ngpu - 1) // ngpu)
    dil = args.open_loop_dilate or float(lpg)
    wl = dataclasses.replace(base, jobs=[dataclasses.replace(j, arrival_ns=int(j.arrival_ns * dil))
                                         for j in base.jobs])
    need_in, need_out = {}, {}
    for sp in wl.jobs:
        need_in[sp.tenant] = [max(a, b) for a, b in zip(need_in.get(sp.tenant, [0, 0]), (sp.h2d_sizes() + [0])[:2])]
        need_out[sp.tenant] = max(need_out.get(sp.tenant, 0), sum(sp.d2h_sizes()))
    hin = {t: [torch.empty(max(1, b), dtype=torch.uint8).pin_memory() for b in v] for t, v in need_in.items()}
    hout = {t: torch.empty(max(1, b), dtype=torch.uint8).pin_memory() for t, b in need_out.items()}
    refs = [([S.HostRef(hin[sp.tenant][i].data_ptr(), b) for i, b in enumerate(sp.h2d_sizes())],
             [S.HostRef(hout[sp.tenant].data_ptr(), b) for b in sp.d2h_sizes()]) for sp in wl.jobs]
    tstar, terms = tstar_device(wl, link, peaks["hbm_gbs"], peaks["bf16_tflops_sustained"] or peaks["bf16_tflops"],
                                kl_slots=lpg * wl.config.partitions)
    variants = [("LAS admission + GUF / LAS (C4)", wl.config.resolved()),
                ("arrival order + GMin / FIFO", dataclasses.replace(wl.config, balancer=W.GMIN, las_admission=0,
                                                                    device_policy=W.FIFO).resolved())]
    weight_of = {t: ten.weight for t, ten in enumerate(wl.tenants)}
    # Third row: the same scheduler in INJECTED timing on the undilated arrivals --
    # decisions in virtual time with the nominal per-device phase durations
    # (SURVEY §8(d)), i.e. the latencies an 8-device box at nominal rates would
    # see; every op still runs on the GPU.
    variants.append(("LAS admission + GUF / LAS (C4), INJECTED virtual time, 8 devices at nominal rates",
                     wl.config.resolved()))
    for vi, (name, cfg) in enumerate(variants):
        injected = vi == 2
        run_wl = base if injected else wl
        with ClockSampler(torch.cuda.current_device()) as clk:
            S.init_from_config(cfg, timing_mode=S.INJECTED if injected else S.MEASURED, physical_gpus=ngpu,
                               trace_in_memory=False)
            ts = [S.register_tenant(t.weight, t.max_inflight) for t in wl.tenants]
            late = []
            ids = [None] * len(wl.jobs)

            def submitter():
                if injected:               # arrival_ns is virtual: submit everything, then drain
                    for i, sp in enumerate(base.jobs):
                        ids[i] = S.submit_spec(ts[sp.tenant], sp, refs[i][0], refs[i][1])
                        late.append(0)
                    return
                t0 = time.perf_counter_ns()
                for i, sp in enumerate(wl.jobs):
                    due = t0 + sp.arrival_ns
                    while time.perf_counter_ns() < due:
                        pass
                    late.append(time.perf_counter_ns() - due)
                    ids[i] = S.submit_spec(ts[sp.tenant], sp, refs[i][0], refs[i][1])

            th = threading.Thread(target=submitter)
            th.start()
            th.join()
            st = S.drain()
            infos = [S.job_info(j) for j in ids]
            S.shutdown()
        dump = os.environ.get("BENCH_OPEN_LOOP_DUMP")
        if dump:                           # per-job records for offline analysis
            with open(f"{dump}.{vi}.jsonl", "w") as f:
                for sp, inf in zip(run_wl.jobs, infos):
                    f.write(json.dumps({"tenant": sp.tenant, "cls": W.CLASS_NAMES[sp.kclass], "gid": inf.gid,
                                        "arr": inf.t_arrival, "place": inf.t_place, "start": list(inf.t_start),
                                        "done": list(inf.t_done)}) + "\n")
        lat, slow = {}, {}
        for sp, inf in zip(run_wl.jobs, infos):
            lat.setdefault(weight_of[sp.tenant], []).append((inf.t_done[2] - inf.t_arrival) / 1e6)
            # slowdown: latency / the job's nominal solo chain (H2D + KL + D2H at the injected
            # rates), so classes with different job mixes compare
            solo = max(1, sp.inj_h2d_ns + sp.inj_kl_ns + sp.inj_d2h_ns)
            slow.setdefault(weight_of[sp.tenant], []).append((inf.t_done[2] - inf.t_arrival) / solo)
        per_class = {f"w={w}": {"jobs": len(v), "p50_ms": round(_pct(v, 0.5), 3), "p99_ms": round(_pct(v, 0.99), 3),
                                "mean_ms": round(sum(v) / len(v), 3),
                                "slowdown_mean": round(sum(slow[w]) / len(slow[w]), 2),
                                "slowdown_p99": round(_pct(slow[w], 0.99), 2)}
                     for w, v in sorted(lat.items(), reverse=True)}
        busy, first, last = {}, {}, {}
        for inf in infos:
            busy[inf.tenant] = busy.get(inf.tenant, 0) + sum(inf.t_done[x] - inf.t_start[x] for x in range(3))
            first[inf.tenant] = min(first.get(inf.tenant, inf.t_arrival), inf.t_arrival)
            last[inf.tenant] = max(last.get(inf.tenant, 0), inf.t_done[2])
        xs = [busy[t] / max(1, last[t] - first[t]) / wl.tenants[t].weight for t in busy]
        jain = sum(xs) ** 2 / (len(xs) * sum(x * x for x in xs))
        span = (max(i.t_done[2] for i in infos) - min(i.t_arrival for i in infos)) / 1e9
        print(json.dumps({"config": f"{args.open_loop_config} open loop", "scheduler": name, "status": st,
                          "failed_jobs": sum(1 for i in infos if i.status != S.OK),
                          "jobs": len(wl.jobs), "logical_gpus": cfg.num_gpus, "physical_gpus": ngpu,
                          "timing": "INJECTED (virtual)" if injected else "MEASURED",
                          "arrival_dilation": 1.0 if injected else dil, "rho_per_device": 0.9,
                          "jobs_per_s": round(len(wl.jobs) / span, 1), "span_ms": round(span * 1e3, 2),
                          "last_arrival_ms": round(run_wl.jobs[-1].arrival_ns / 1e6, 2),
                          "tstar_ms": None if injected else round(tstar * 1e3, 3),
                          "roofline_frac": None if injected else round(tstar / span, 4),
                          "tstar_terms_ms": None if injected else {k: round(v * 1e3, 3) for k, v in terms.items()},
                          "latency_by_priority": per_class,
                          "latency_all": {"p50_ms": round(_pct([x for v in lat.values() for x in v], 0.5), 3),
                                          "p99_ms": round(_pct([x for v in lat.values() for x in v], 0.99), 3)},
                          "jain_weighted_service": round(jain, 4),
                          "submit_lateness_us": {"p50": round(_pct(late, 0.5) / 1e3, 1),
                                                 "p99": round(_pct(late, 0.99) / 1e3, 1),
                                                 "max": round(max(late) / 1e3, 1)},
                          "clocks": clk.summary(),
                          "note": "latency = JOB_DONE - arrival; priority class = tenant weight; " + (
                              "virtual clock: each logical device has its own nominal engines" if injected else
                              "logical devices share the physical GPU's host link and SMs"
                              if cfg.num_gpus > ngpu else "one logical device per GPU")}), flush=True)
    del hin, hout


def main():
    args = parse_args()
    if args.open_loop:
        open_loop(args)
        return
    if args.configs:
        run_configs(args)
        return
    if args.fig2:
        fig2(args)
        return
    if args.sweep:
        policy_sweep(args)
        return
    from paper_conf_sc_senguptagsp14_b200 import parallel as par
    info = par.rank_info()
    world, rank = info.world, info.rank
    if args.impl == "reference":
        if rank == 0:
            run_reference(args)
        return
    if args.gpus > 1 or world > 1:
        # N GPUs: node mode -- rank 0 owns every GPU through the level-1 balancer
        args.gpus = max(args.gpus, world)
        gloo = par.init_groups(info, device_backend=None, timeout_s=4 * 3600)

        def work(group):
            import torch
            res, _ = run_node(args, torch, group, world)
            res["paper_context"] = PAPER_CONTEXT
            print(json.dumps(res), flush=True)
            return res
        par.node_mode(info, gloo, work)
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()
        return
    par.isolate_gpu(info)                 # one process per GPU (before CUDA init)
    numa = par.bind_to_gpu_numa_node(par.physical_gpu(info))
    if world > 1 and "STRINGS_COPY_THREADS" not in os.environ:
        # ranks bound to the same CPUs share them: each rank's PMT copy pool gets its share
        os.environ["STRINGS_COPY_THREADS"] = str(par.copy_threads_per_rank(info))
        numa["copy_threads"] = int(os.environ["STRINGS_COPY_THREADS"])
    import torch
    gloo = par.init_groups(info, device_backend="nccl")
    res, wl = run_strings(args, rank, world, torch, gloo)
    if rank == 0:
        res["config"]["host_numa"] = numa
        res["paper_context"] = PAPER_CONTEXT
        if world == 1 and not args.no_static:
            from paper_conf_sc_senguptagsp14_b200.static_baseline import run_static
            sb = run_static(wl, num_gpus=1, repeats=args.static_repeats)
            sb["note"] = "at N = 1 'tenant mod N' and 'device 0' are the same placement"
            res["static_baseline"] = sb
            res["speedup_vs_static"] = round(res["value"] / sb["value"], 3)
            # weighted speedup, Eq. (2) (reading R-1): mean over tenants of
            # mean latency under static provisioning / under Strings
            mine = res.pop("_mean_latency_s_by_tenant")
            st = sb["mean_latency_s_by_tenant"]
            ws = sum(st[t] / mine[t] for t in mine) / len(mine)
            res["weighted_speedup_vs_static"] = round(ws, 3)
        res.pop("_mean_latency_s_by_tenant", None)
        if world == 1:
            res["cpu_baseline"] = cpu_baseline(wl)
        print(json.dumps(res), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
