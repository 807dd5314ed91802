"""Seeded synthetic workloads for the Strings scheduler (inputs only).

This module is shared by the oracle (``oracle/``) and the CUDA path
(``paper_conf_sc_senguptagsp14_b200``).  It holds NO arithmetic of the method:
no scheduling decision, no service accounting, no balancer score, no tenant
kernel.  It only produces inputs:

* the tenant list (weights, in-flight limits),
* the job list (class, sizes, arrival time, priority, injected phase
  durations, data seed), and
* the input data of each job (fp32 vectors, bf16 matrices, u32 vectors).

Arrival times follow the paper's negative-exponential inter-arrival model,
Eq. (4) (§V.C): ``T = -lambda * ln(X)``, ``X in (0, 1]``.
The formula glyphs are lost in PAPER.md; reading R-3 restates it.
X is drawn from SplitMix64 so that the stream is bit-identical everywhere;
arrival times are floored to integer ns once, here, so libm never reaches a
scheduler decision.

Injected phase durations are inputs as well: they are the
per-phase times the virtual clock uses in INJECTED timing mode, derived from
the job's bytes at fixed nominal rates so that traces never drift when the
hardware is re-measured.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field, asdict
from typing import List, Optional

import numpy as np

# ----------------------------------------------------------------------------
# Enumerations (numeric values are part of the C ABI, include/strings_sched.h)
# ----------------------------------------------------------------------------
VSCALE, GEMM, XFER, HIST, SCAN, SORT = 0, 1, 2, 3, 4, 5
CLASS_NAMES = {VSCALE: "VSCALE", GEMM: "GEMM", XFER: "XFER", HIST: "HIST", SCAN: "SCAN", SORT: "SORT"}
SORT_SEGMENT = 2048

GRR, GMIN, GWTMIN, RTF, GUF, DTF, MBF, DYNAMIC = range(8)
BALANCER_NAMES = ["GRR", "GMIN", "GWTMIN", "RTF", "GUF", "DTF", "MBF", "DYNAMIC"]
FIFO, LAS, PS, TFS = 0, 1, 2, 3
DEVICE_POLICY_NAMES = ["FIFO", "LAS", "PS", "TFS"]

# Nominal rates used ONLY to make injected durations (inputs).  Integer
# bytes/ns and FLOP/ns; see DESIGN.md §5 "Injected durations".
INJ_LINK_BYTES_PER_NS = 50          # 50 GB/s per copy direction
INJ_HBM_BYTES_PER_NS = 6000         # 6 TB/s
INJ_KL_FLOP_PER_NS = 700_000        # 700 TFLOP/s for one KL slot


def _ceil_div(a: int, b: int) -> int:
    return -(-a // b)


# ----------------------------------------------------------------------------
# SplitMix64 (Steele, Lea, Flood 2014) -- integer generator, bit-identical
# ----------------------------------------------------------------------------
_MASK64 = (1 << 64) - 1


class SplitMix64:
    def __init__(self, seed: int):
        self.state = seed & _MASK64

    def next_u64(self) -> int:
        self.state = (self.state + 0x9E3779B97F4A7C15) & _MASK64
        z = self.state
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _MASK64
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _MASK64
        return z ^ (z >> 31)

    def unit_open0(self) -> float:
        """X in (0, 1]: (u53 + 1) * 2^-53 (reading R-3)."""
        return ((self.next_u64() >> 11) + 1) * (1.0 / (1 << 53))


def exp_interarrival_ns(rng: SplitMix64, lam_ns: float) -> int:
    """One inter-arrival gap, Eq. (4): T = -lambda*ln(X)."""
    x = rng.unit_open0()
    return int(math.floor(-lam_ns * math.log(x)))


# ----------------------------------------------------------------------------
# Workload description
# ----------------------------------------------------------------------------
@dataclass
class TenantSpec:
    weight: int = 1
    max_inflight: int = 1


@dataclass
class JobSpec:
    tenant: int
    kclass: int
    n: int = 0            # VSCALE/XFER length; GEMM N
    m: int = 0            # GEMM M
    k: int = 0            # GEMM K
    reps: int = 1         # GEMM repetitions R
    alpha: float = 1.0    # VSCALE scalar (fp32)
    seed: int = 0         # XFER seed
    data_seed: int = 0    # seed of this job's input data
    int_valued: bool = False  # GEMM: integer-valued operands in [-2, 2]
    arrival_ns: int = 0
    priority: int = 0     # 0 -> tenant weight
    inj_h2d_ns: int = 0
    inj_kl_ns: int = 0
    inj_d2h_ns: int = 0

    # Buffer sizes (bytes).  The H2D buffers of a job are, in order:
    #   VSCALE: x[n] fp32;  GEMM: A[m*k] bf16, B[k*n] bf16;  XFER/SCAN/SORT: x[n] u32;
    #   HIST: x[n] u8
    # and its D2H buffer is y[n] fp32 / C[m*n] fp32 / y[n] u32 / bins[256] u32.
    def h2d_sizes(self) -> List[int]:
        if self.kclass == GEMM:
            return [2 * self.m * self.k, 2 * self.k * self.n]
        if self.kclass == HIST:
            return [self.n]
        return [4 * self.n]

    def d2h_sizes(self) -> List[int]:
        if self.kclass == GEMM:
            return [4 * self.m * self.n]
        if self.kclass == HIST:
            return [1024]
        return [4 * self.n]


@dataclass
class SystemConfig:
    num_gpus: int = 1          # G logical devices
    balancer: int = GMIN
    las_admission: int = 0
    device_policy: int = PS
    partitions: int = 2        # P KL slots per device
    awake_budget: int = 0      # A (0 -> 2 + P)
    admit_cap: int = 0         # M (0 -> 2 * A)
    quantum_ns: int = 1_000_000
    joint_select: int = -1     # -1 auto (on for DTF/MBF/DYNAMIC)
    tfs_slice_ns: int = 500_000  # TFS base slice S (a tenant of weight w is awake for w*S of service)
    device_weights: Optional[List[int]] = None   # DST weights per logical device (None = all 1)

    def resolved(self) -> "SystemConfig":
        c = SystemConfig(**asdict(self))
        if c.awake_budget <= 0:
            c.awake_budget = 2 + c.partitions
        if c.admit_cap <= 0:
            c.admit_cap = 2 * c.awake_budget
        if c.joint_select < 0:
            c.joint_select = 1 if c.balancer in (DTF, MBF, DYNAMIC) else 0
        if c.device_weights is None:
            c.device_weights = [1] * c.num_gpus
        return c


@dataclass
class Workload:
    name: str
    config: SystemConfig
    tenants: List[TenantSpec]
    jobs: List[JobSpec]          # in submission order (job id = index)
    notes: str = ""

    def sorted_check(self) -> None:
        last = {}
        for j in self.jobs:
            assert j.arrival_ns >= last.get(j.tenant, 0), "per-tenant arrivals must be nondecreasing"
            last[j.tenant] = j.arrival_ns


# ----------------------------------------------------------------------------
# Injected durations (inputs; nominal integer rates)
# ----------------------------------------------------------------------------
def nominal_durations(j: JobSpec) -> tuple:
    h2d = sum(j.h2d_sizes())
    d2h = sum(j.d2h_sizes())
    kl_flop = 0
    if j.kclass == GEMM:
        kl_bytes = 2 * j.m * j.k + 2 * j.k * j.n + 4 * j.m * j.n
        kl_flop = 2 * j.m * j.n * j.k * j.reps
    elif j.kclass == HIST:
        kl_bytes = j.n + 1024
    else:
        kl_bytes = 8 * j.n
    kl = max(_ceil_div(kl_bytes, INJ_HBM_BYTES_PER_NS), _ceil_div(kl_flop, INJ_KL_FLOP_PER_NS))
    return (_ceil_div(h2d, INJ_LINK_BYTES_PER_NS), kl, _ceil_div(d2h, INJ_LINK_BYTES_PER_NS))


def with_nominal_durations(j: JobSpec) -> JobSpec:
    j.inj_h2d_ns, j.inj_kl_ns, j.inj_d2h_ns = nominal_durations(j)
    return j


# ----------------------------------------------------------------------------
# Job input data (seeded)
# ----------------------------------------------------------------------------
def f32_to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """fp32 -> bf16 bit pattern, round-to-nearest-even (inputs have no NaN)."""
    u = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    rounding = 0x7FFF + ((u >> 16) & 1)
    return ((u + rounding) >> 16).astype(np.uint16)


def job_inputs(j: JobSpec) -> List[np.ndarray]:
    """The H2D buffers of job j, in order, as numpy arrays (C-contiguous)."""
    rng = np.random.Generator(np.random.PCG64(j.data_seed))
    if j.kclass == VSCALE:
        return [rng.uniform(-1.0, 1.0, size=j.n).astype(np.float32)]
    if j.kclass in (XFER, SCAN, SORT):
        return [rng.integers(0, 1 << 32, size=j.n, dtype=np.uint64).astype(np.uint32)]
    if j.kclass == HIST:
        # image-like bytes: a skewed mixture (a few hot bins + uniform background)
        hot = rng.integers(0, 256, size=8)
        pick = rng.integers(0, 4, size=j.n)
        vals = np.where(pick == 0, hot[rng.integers(0, 8, size=j.n)], rng.integers(0, 256, size=j.n))
        return [vals.astype(np.uint8)]
    if j.kclass == GEMM:
        if j.int_valued:
            a = rng.integers(-2, 3, size=(j.m, j.k)).astype(np.float32)
            b = rng.integers(-2, 3, size=(j.k, j.n)).astype(np.float32)
        else:
            a = rng.uniform(-1.0, 1.0, size=(j.m, j.k)).astype(np.float32)
            b = rng.uniform(-1.0, 1.0, size=(j.k, j.n)).astype(np.float32)
        return [f32_to_bf16_bits(a), f32_to_bf16_bits(b)]
    raise ValueError(f"unknown class {j.kclass}")


def job_output_shapes(j: JobSpec) -> List[tuple]:
    if j.kclass == GEMM:
        return [((j.m, j.n), np.float32)]
    if j.kclass == VSCALE:
        return [((j.n,), np.float32)]
    if j.kclass == HIST:
        return [((256,), np.uint32)]
    return [((j.n,), np.uint32)]


# ----------------------------------------------------------------------------
# The five BASELINE.json configurations and small variants
# ----------------------------------------------------------------------------
VSCALE_N = 1 << 20          # "1M floats" (reading R-21: 2^20)
GEMM_DIM = 256
XFER_N = 1 << 24            # 64 MiB of u32


def _vscale(t, ds, n=VSCALE_N):
    return JobSpec(tenant=t, kclass=VSCALE, n=n, alpha=1.0 + 2.0 ** -10, data_seed=ds)


def _gemm(t, ds, reps=64, dim=GEMM_DIM, int_valued=False):
    return JobSpec(tenant=t, kclass=GEMM, m=dim, n=dim, k=dim, reps=reps, data_seed=ds,
                   int_valued=int_valued)


def _xfer(t, ds, n=XFER_N):
    return JobSpec(tenant=t, kclass=XFER, n=n, seed=(0x9E3779B9 * (t + 1)) & 0xFFFFFFFF,
                   data_seed=ds)


def _closed_loop(name, cfg, tenants, per_tenant_jobs, maker, notes=""):
    """All jobs arrive at t=0; tenant t's jobs are submitted round-robin."""
    jobs = []
    for s in range(per_tenant_jobs):
        for t in range(len(tenants)):
            jobs.append(with_nominal_durations(maker(t, s)))
    return Workload(name, cfg, tenants, jobs, notes)


def config_c1(seed: int = 1, reps: int = 64, scale: int = 1, int_valued: bool = False) -> Workload:
    """C1: 4 tenants (2 VSCALE 1M floats, 2 GEMM 256^3) x 8 requests, 2 GPUs, PS."""
    cfg = SystemConfig(num_gpus=2, balancer=GMIN, device_policy=PS)
    tenants = [TenantSpec() for _ in range(4)]

    def mk(t, s):
        ds = seed * 1_000_003 + t * 1009 + s
        if t < 2:
            return _vscale(t, ds, n=VSCALE_N // scale)
        return _gemm(t, ds, reps=reps, int_valued=int_valued)
    return _closed_loop("C1", cfg, tenants, 8, mk)


def config_c2(seed: int = 1, reps: int = 64, scale: int = 1, jobs_per_tenant: int = 8,
              num_gpus: int = 1) -> Workload:
    """C2: 16 tenants (8 GEMM R=64 + 8 XFER), 1 GPU, DTF (joint selection).
    num_gpus = N > 1 is the weak-scaled variant the bench runs at N GPUs: 16N
    tenants of the same mix (16 per GPU), placed by the balancer."""
    cfg = SystemConfig(num_gpus=num_gpus, balancer=DTF, device_policy=PS)
    tenants = [TenantSpec() for _ in range(16 * num_gpus)]

    def mk(t, s):
        ds = seed * 1_000_003 + t * 1009 + s
        if t % 2 == 0:
            return _gemm(t, ds, reps=reps)
        return _xfer(t, ds, n=XFER_N // scale)
    return _closed_loop("C2", cfg, tenants, jobs_per_tenant, mk)


def config_c3(seed: int = 1, reps: int = 64, scale: int = 1) -> Workload:
    """C3: 32 tenants = 16 VSCALE + 16 GEMM pairs, 4 GPUs, MBF."""
    cfg = SystemConfig(num_gpus=4, balancer=MBF, device_policy=PS)
    tenants = [TenantSpec() for _ in range(32)]

    def mk(t, s):
        ds = seed * 1_000_003 + t * 1009 + s
        if t % 2 == 0:
            return _vscale(t, ds, n=VSCALE_N // scale)
        return _gemm(t, ds, reps=reps)
    return _closed_loop("C3", cfg, tenants, 8, mk)


def config_c4(seed: int = 1, reps: int = 64, scale: int = 1, rho: float = 0.9,
              jobs_per_tenant: int = 32) -> Workload:
    """C4: 64 tenants, Poisson arrivals (Eq. 4), skewed priorities, 8 GPUs,
    LAS admission + GUF placement, LAS device policy."""
    cfg = SystemConfig(num_gpus=8, balancer=GUF, las_admission=1, device_policy=LAS)
    weights = [8] * 4 + [4] * 8 + [2] * 16 + [1] * 36
    tenants = [TenantSpec(weight=w) for w in weights]
    per_tenant = []
    for t in range(64):
        row = []
        for s in range(jobs_per_tenant):
            ds = seed * 1_000_003 + t * 1009 + s
            c = t % 3
            j = _vscale(t, ds, VSCALE_N // scale) if c == 0 else (
                _gemm(t, ds, reps=reps) if c == 1 else _xfer(t, ds, XFER_N // scale))
            row.append(with_nominal_durations(j))
        per_tenant.append(row)
    # lambda_t = T_solo_t * 64 / (8 * rho): offered load ~rho per device.
    rng = SplitMix64(0x5EED0000 + seed)
    for t in range(64):
        j0 = per_tenant[t][0]
        t_solo = max(j0.inj_h2d_ns, j0.inj_kl_ns, j0.inj_d2h_ns)
        lam = t_solo * 64.0 / (8.0 * rho)
        now = 0
        for j in per_tenant[t]:
            now += exp_interarrival_ns(rng, lam)
            j.arrival_ns = now
    jobs = sorted((j for row in per_tenant for j in row), key=lambda j: (j.arrival_ns, j.tenant))
    return Workload("C4", cfg, tenants, jobs)


def config_c5(seed: int = 1, reps: int = 64, scale: int = 1, jobs_per_tenant: int = 24) -> Workload:
    """C5: 128 tenants, phase-changing classes (rotate every 4 jobs), 8 GPUs, DYNAMIC."""
    cfg = SystemConfig(num_gpus=8, balancer=DYNAMIC, device_policy=PS)
    tenants = [TenantSpec() for _ in range(128)]

    def mk(t, s):
        ds = seed * 1_000_003 + t * 1009 + s
        c = ((s // 4) + t) % 3
        if c == 0:
            return _vscale(t, ds, VSCALE_N // scale)
        if c == 1:
            return _gemm(t, ds, reps=reps)
        return _xfer(t, ds, XFER_N // scale)
    return _closed_loop("C5", cfg, tenants, jobs_per_tenant, mk)


def config_c4c(seed: int = 1, reps: int = 64, scale: int = 1, jobs_per_tenant: int = 32) -> Workload:
    """C4 under admission contention (not a BASELINE.json config; the variant
    that exercises LAS at the balancer): the same 64 tenants
    and skewed weights, offered twice the box's capacity (rho = 2.0), each
    tenant with c_t = 4 requests in flight, at most M = 4 resident jobs per
    device -- so admissions queue and the weighted-LAS order decides who goes
    next."""
    wl = config_c4(seed=seed, reps=reps, scale=scale, rho=2.0, jobs_per_tenant=jobs_per_tenant)
    for t in wl.tenants:
        t.max_inflight = 4
    wl.config.admit_cap = 4
    wl.name = "C4c"
    return wl


CONFIGS = {"C1": config_c1, "C2": config_c2, "C3": config_c3, "C4": config_c4, "C5": config_c5,
           "C4c": config_c4c}

# ----------------------------------------------------------------------------
# NEXT-2: the paper's pairwise mix (6 long x 4 short apps -> 24
# pairs A..X in Table I order).  Here: long = {GEMM (MM), HIST (HI), SCAN (SC)},
# short = {VSCALE (BS-like streaming), XFER (MC-like transfer-heavy), SORT (SN)}
# -> 9 pairs A..I.  Each pair runs `instances` tenants of each app, requests
# arriving by Eq. (4) with lambda proportional to the app's runtime (L885-889).
# ----------------------------------------------------------------------------
PAIR_LONG = ("GEMM", "HIST", "SCAN")
PAIR_SHORT = ("VSCALE", "XFER", "SORT")
PAIRS = [(a, b) for a in PAIR_LONG for b in PAIR_SHORT]          # A..I


def _pair_job(cls: str, t: int, ds: int, scale: int) -> JobSpec:
    if cls == "GEMM":
        return _gemm(t, ds, reps=256)
    if cls == "HIST":
        return JobSpec(tenant=t, kclass=HIST, n=(1 << 26) // scale, data_seed=ds)
    if cls == "SCAN":
        return JobSpec(tenant=t, kclass=SCAN, n=(1 << 24) // scale, data_seed=ds)
    if cls == "VSCALE":
        return _vscale(t, ds, n=VSCALE_N // scale)
    if cls == "XFER":
        return _xfer(t, ds, n=(1 << 22) // scale)
    if cls == "SORT":
        return JobSpec(tenant=t, kclass=SORT, n=max(SORT_SEGMENT, (1 << 20) // scale), data_seed=ds)
    raise ValueError(cls)


def config_pair(index: int, seed: int = 1, num_gpus: int = 2, balancer: int = GMIN, instances: int = 4,
                jobs_per_tenant: int = 8, load: float = 0.8, scale: int = 1) -> Workload:
    """Pair `index` (0 = 'A' ...) of the pairwise mix."""
    a, b = PAIRS[index]
    cfg = SystemConfig(num_gpus=num_gpus, balancer=balancer, device_policy=PS)
    tenants = [TenantSpec() for _ in range(2 * instances)]
    rng = SplitMix64(0xA11CE + 97 * index + seed)
    jobs = []
    for t in range(2 * instances):
        cls = a if t % 2 == 0 else b
        now = 0
        for s in range(jobs_per_tenant):
            j = with_nominal_durations(_pair_job(cls, t, seed * 1_000_003 + t * 1009 + s, scale))
            t_solo = max(j.inj_h2d_ns, j.inj_kl_ns, j.inj_d2h_ns)
            # per-tenant rate: the pair's 2*instances tenants share num_gpus devices at `load`
            lam = t_solo * (2 * instances) / (num_gpus * load)
            now += exp_interarrival_ns(rng, lam)
            j.arrival_ns = now
            jobs.append(j)
    jobs.sort(key=lambda j: (j.arrival_ns, j.tenant))
    return Workload(f"pair-{chr(65 + index)}:{a}-{b}", cfg, tenants, jobs)


def random_workload(seed: int, max_gpus: int = 3, max_tenants: int = 6, max_jobs: int = 24,
                    tiny: bool = True) -> Workload:
    """A random small workload for differential/invariant tests (tiny sizes)."""
    r = np.random.Generator(np.random.PCG64(seed))
    cfg = SystemConfig(
        num_gpus=int(r.integers(1, max_gpus + 1)),
        balancer=int(r.integers(0, 8)),
        las_admission=int(r.integers(0, 2)),
        device_policy=int(r.integers(0, 4)),
        partitions=int(r.integers(1, 4)),
        quantum_ns=int(r.choice([1_000, 7_919, 100_000, 1_000_000])),
    )
    if r.integers(0, 3) == 0:
        cfg.awake_budget = int(r.integers(1, 6))
    if r.integers(0, 3) == 0:
        cfg.admit_cap = int(r.integers(1, 8))
    if r.integers(0, 2) == 0:
        cfg.joint_select = int(r.integers(0, 2))
    if cfg.device_policy == TFS:
        cfg.tfs_slice_ns = int(r.choice([1, 5_000, 100_000, 500_000]))
    if r.integers(0, 3) == 0:
        cfg.device_weights = [int(x) for x in r.integers(1, 4, cfg.num_gpus)]
    T = int(r.integers(1, max_tenants + 1))
    tenants = [TenantSpec(weight=int(r.integers(1, 9)), max_inflight=int(r.integers(1, 4)))
               for _ in range(T)]
    njobs = int(r.integers(1, max_jobs + 1))
    arrivals = {t: 0 for t in range(T)}
    jobs = []
    for i in range(njobs):
        t = int(r.integers(0, T))
        c = int(r.integers(0, 6))
        ds = seed * 7919 + i
        if c == VSCALE:
            j = JobSpec(tenant=t, kclass=VSCALE, n=int(r.choice([0, 1, 5, 1024, 4099])) if tiny else VSCALE_N,
                        alpha=float(np.float32(r.uniform(-2, 2))), data_seed=ds)
        elif c == GEMM:
            j = JobSpec(tenant=t, kclass=GEMM, m=128, n=256, k=int(r.choice([64, 128, 256])),
                        reps=int(r.integers(1, 5)), data_seed=ds, int_valued=bool(r.integers(0, 2)))
        elif c == XFER:
            j = JobSpec(tenant=t, kclass=XFER, n=int(r.choice([0, 3, 4096, 65537])) if tiny else XFER_N,
                        seed=int(r.integers(0, 1 << 32)), data_seed=ds)
        elif c == HIST:
            j = JobSpec(tenant=t, kclass=HIST, n=int(r.choice([0, 1, 17, 4096, 100_003])), data_seed=ds)
        elif c == SCAN:
            j = JobSpec(tenant=t, kclass=SCAN, n=int(r.choice([0, 1, 9, 2047, 70_001])), data_seed=ds)
        else:
            j = JobSpec(tenant=t, kclass=SORT, n=SORT_SEGMENT * int(r.choice([0, 1, 3, 40])), data_seed=ds)
        if r.integers(0, 2):
            arrivals[t] += int(r.choice([0, 0, 1, 500, 20_000, 2_000_000]))
        j.arrival_ns = arrivals[t]
        j.priority = int(r.integers(0, 4))
        with_nominal_durations(j)
        if r.integers(0, 4) == 0:       # occasional zero-length phases
            j.inj_h2d_ns = 0
        if r.integers(0, 4) == 0:
            j.inj_kl_ns = 0
        jobs.append(j)
    return Workload(f"rand{seed}", cfg, tenants, jobs)
