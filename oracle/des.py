"""Deterministic discrete-event model of the Strings two-level scheduler.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
module.  It shares no code with the CUDA path (``paper_conf_sc_senguptagsp14_b200``);
its only common dependency is the seeded input generator ``strings_workload``.

This is the *algorithm, step by step* (SURVEY.md §8(c)): the paper's policies
applied in the paper's order to a virtual clock, with every reading the paper
leaves open taken from DESIGN.md §4 (readings R-n).  It is deliberately plain:
lists, linear scans, no incremental data structures.

Paper passages (PAPER.md line numbers, section):
  GRR            L683  §IV.A.1      next GPU round robin
  GMin           L685-687 §IV.A.2   fewest bound applications, ties -> lowest GID (R-13)
  GWtMin         L689  §IV.A.3      weighted minimum load
  LAS            L693  §IV.B.1      least attained service first (weighted, R-7)
  Eq. (1)        L695               CGS_n = k*GS_n + (1-k)*CGS_{n-1}, k = 0.8 (integer form R-4)
  PS             L819  §IV.B.3      wake threads in different phases, else KL > H2D = D2H > DFL (R-11)
  TFS            L699, L817 §IV.B.2 at most one tenant awake, weight-proportional slices, penalty
                                    for overshoot via weighted service history, work-conserving (R-28)
  RTF/GUF/DTF/MBF L823-831 §IV.C    feedback placement policies (scores R-13)
  Policy arbiter L311, L1073        switch on sufficient feedback (R-15)
  RCB / SFT / DST L309-313, L489-515, Fig 6
  async + per-app order L295-299 §III.B.2 (a tenant's jobs run in submission order)

Outputs: the canonical decision trace, per-job timestamps.
"""
from __future__ import annotations

import functools
import heapq
from dataclasses import dataclass, field
from typing import Dict, List, Optional, Tuple

import strings_workload as W

H2D, KL, D2H = 0, 1, 2
ENGINE_NAMES = ("H2D", "KL", "D2H")
POLICY_NAMES = W.BALANCER_NAMES

# Nominal integer peaks for class priors and MBF decomposition (R-13).
PRIOR_LINK_BYTES_PER_NS = 50
PRIOR_HBM_BYTES_PER_NS = 6000
PRIOR_KL_FLOP_PER_NS = 700_000


def ceil_div(a: int, b: int) -> int:
    return -(-a // b)


def class_hbm_bytes_and_flop(spec: W.JobSpec) -> Tuple[int, int]:
    """Algorithmic kernel bytes and tensor FLOP of one job."""
    if spec.kclass == W.VSCALE:
        return 8 * spec.n, 0                      # read x, write y (fp32)
    if spec.kclass == W.XFER:
        return 8 * spec.n, 0                      # read x, write y (u32)
    if spec.kclass == W.GEMM:
        m, n, k = spec.m, spec.n, spec.k
        return 2 * m * k + 2 * k * n + 4 * m * n, 2 * m * n * k * spec.reps
    if spec.kclass == W.HIST:
        return spec.n + 1024, 0                   # read bytes, write 256 u32 bins
    if spec.kclass in (W.SCAN, W.SORT):
        return 8 * spec.n, 0                      # read x, write y (u32)
    raise ValueError(spec.kclass)


@dataclass
class Job:
    id: int
    spec: W.JobSpec
    tenant: int
    seq: int
    prio: int
    arrival: int
    h2d_bytes: int
    d2h_bytes: int
    hbm_bytes: int
    tflop: int
    dur: Tuple[int, int, int]
    arrived: bool = False
    placed: bool = False
    gid: int = -1
    t_place: int = -1
    place_order: int = -1
    phase: int = 0                 # number of phases DONE (0..3)
    woken: bool = False            # current phase woken (in FIFO or running)
    start: List[int] = field(default_factory=lambda: [-1, -1, -1])
    done: List[int] = field(default_factory=lambda: [-1, -1, -1])
    slot: List[int] = field(default_factory=lambda: [-1, -1, -1])
    t_jobdone: int = -1


@dataclass
class SFTEntry:
    """Scheduler Feedback Table row (Fig 6), per (tenant, class)."""
    count: int = 0
    h2d: int = 0
    kl: int = 0
    d2h: int = 0
    util: int = 0          # Q16


@dataclass
class Device:
    gid: int
    P: int
    resident: List[int] = field(default_factory=list)          # job ids, placement order
    fifo: Tuple[list, list, list] = field(default_factory=lambda: ([], [], []))
    busy: List[List[Optional[int]]] = field(default_factory=list)  # per engine, per slot
    woken_unfinished: int = 0
    weight: int = 1        # DST device weight (L309); equal on identical B200s
    awake: Optional[int] = None          # TFS: the tenant currently awake on this device
    awake_used: int = 0                  # TFS: its service on this device since it woke
    svc: Dict[int, int] = field(default_factory=dict)   # TFS: cumulative service per tenant

    def __post_init__(self):
        self.busy = [[None], [None] * self.P, [None]]


@dataclass
class Tenant:
    weight: int
    c: int                  # max in-flight jobs (server threads, L879)
    pending: List[int] = field(default_factory=list)   # job ids not yet placed, seq order
    inflight: int = 0
    cgs: int = 0            # Q48.16 ns, Eq. (1)
    gs_acc: int = 0         # ns of service in the current epoch (completed parts)


class Oracle:
    def __init__(self, wl: W.Workload):
        self.wl = wl
        cfg = wl.config.resolved()
        self.cfg = cfg
        self.G, self.P, self.A, self.M, self.Q = (cfg.num_gpus, cfg.partitions, cfg.awake_budget,
                                                  cfg.admit_cap, cfg.quantum_ns)
        self.S = cfg.tfs_slice_ns
        assert self.G >= 1 and self.P >= 1 and self.A >= 1 and self.M >= 1 and self.Q >= 1
        self.tenants = [Tenant(weight=t.weight, c=t.max_inflight) for t in wl.tenants]
        self.jobs: List[Job] = []
        seqs: Dict[int, int] = {}
        for i, s in enumerate(wl.jobs):
            seq = seqs.get(s.tenant, 0)
            seqs[s.tenant] = seq + 1
            hbm, fl = class_hbm_bytes_and_flop(s)
            self.jobs.append(Job(
                id=i, spec=s, tenant=s.tenant, seq=seq,
                prio=s.priority if s.priority > 0 else wl.tenants[s.tenant].weight,
                arrival=s.arrival_ns, h2d_bytes=sum(s.h2d_sizes()), d2h_bytes=sum(s.d2h_sizes()),
                hbm_bytes=hbm, tflop=fl, dur=(s.inj_h2d_ns, s.inj_kl_ns, s.inj_d2h_ns)))
            self.tenants[s.tenant].pending.append(i)
        self.devices = [Device(gid=d, P=self.P, weight=cfg.device_weights[d]) for d in range(self.G)]
        self.sft: Dict[Tuple[int, int], SFTEntry] = {}
        self.arrival_order = sorted(range(len(self.jobs)),
                                    key=lambda i: (self.jobs[i].arrival, self.jobs[i].tenant, self.jobs[i].seq))
        self.next_arrival = 0
        self.done_heap: list = []          # (t, gid, engine, slot, job)
        self.epoch_start = 0
        self.next_epoch = self.Q
        self.grr_cursor = 0
        self.place_counter = 0
        self.jobs_done = 0
        self.trace: List[str] = []

    # ------------------------------------------------------------------ trace
    def rec(self, t, kind, gid=None, eng=None, slot=None, tenant=None, seq=None, job=None,
            a1=0, a2=0):
        f = lambda v: "-" if v is None else str(v)
        e = "-" if eng is None else ENGINE_NAMES[eng]
        self.trace.append(f"{t} {kind} {f(gid)} {e} {f(slot)} {f(tenant)} {f(seq)} {f(job)} {a1} {a2}")

    # ------------------------------------------------------------ LAS ordering
    def las_cmp(self, a: Job, b: Job) -> int:
        """Weighted LAS (L693, R-7): a before b iff CGS_a * p_b < CGS_b * p_a;
        ties -> lower tenant -> lower seq."""
        ca, cb = self.tenants[a.tenant].cgs, self.tenants[b.tenant].cgs
        lhs, rhs = ca * b.prio, cb * a.prio
        if lhs != rhs:
            return -1 if lhs < rhs else 1
        if a.tenant != b.tenant:
            return -1 if a.tenant < b.tenant else 1
        return (a.seq > b.seq) - (a.seq < b.seq)

    def las_key_less(self, a: Job, b: Job) -> bool:
        """Strict weighted-key order only (no tenant/seq tie-break)."""
        return self.tenants[a.tenant].cgs * b.prio < self.tenants[b.tenant].cgs * a.prio

    def las_sorted(self, js: List[Job]) -> List[Job]:
        return sorted(js, key=functools.cmp_to_key(self.las_cmp))

    def admission_sorted(self, js: List[Job]) -> List[Job]:
        if self.cfg.las_admission:
            return self.las_sorted(js)
        return sorted(js, key=lambda j: (j.arrival, j.tenant, j.seq))

    # -------------------------------------------------------------- predictions
    def pred(self, j: Job) -> Tuple[int, int, int, int]:
        """(h2d, kl, d2h, util_q16): SFT EWMAs if (tenant, class) has a sample,
        else the class prior at nominal peaks (R-13)."""
        e = self.sft.get((j.tenant, j.spec.kclass))
        if e is not None and e.count > 0:
            return e.h2d, e.kl, e.d2h, e.util
        h = ceil_div(j.h2d_bytes, PRIOR_LINK_BYTES_PER_NS)
        d = ceil_div(j.d2h_bytes, PRIOR_LINK_BYTES_PER_NS)
        k = max(ceil_div(j.hbm_bytes, PRIOR_HBM_BYTES_PER_NS), ceil_div(j.tflop, PRIOR_KL_FLOP_PER_NS))
        tot = h + k + d
        return h, k, d, (k * 65536 // tot) if tot else 0

    def has_sample(self, j: Job) -> bool:
        e = self.sft.get((j.tenant, j.spec.kclass))
        return e is not None and e.count > 0

    def effective_policy(self, j: Job) -> int:
        """Policy arbiter (L311, L1073; R-15): feedback policies need >= 1 sample."""
        b = self.cfg.balancer
        if b in (W.RTF, W.GUF, W.DTF, W.MBF, W.DYNAMIC) and not self.has_sample(j):
            return W.GMIN
        if b == W.DYNAMIC:
            return W.MBF
        return b

    # ------------------------------------------------------------------ scores
    def score(self, policy: int, j: Job, d: Device) -> int:
        """Balancer score of placing j on d (minimised; R-13)."""
        res = [self.jobs[i] for i in d.resident]
        if policy in (W.GMIN, W.GWTMIN):
            return len(res)
        if policy == W.RTF:                         # L823-825: predicted remaining runtime
            s = 0
            for i in res:
                h, k, dd, _ = self.pred(i)
                s += (h if i.phase <= H2D else 0) + (k if i.phase <= KL else 0) + (dd if i.phase <= D2H else 0)
            h, k, dd, _ = self.pred(j)
            return s + h + k + dd
        if policy == W.GUF:                         # L827: sum of GPU utilisation
            return sum(self.pred(i)[3] for i in res) + self.pred(j)[3]
        if policy == W.DTF:                         # L829: balance transfer vs compute time
            copy = kern = 0
            for i in res:
                h, k, dd, _ = self.pred(i)
                copy += (h if i.phase <= H2D else 0) + (dd if i.phase <= D2H else 0)
                kern += k if i.phase <= KL else 0
            h, k, dd, _ = self.pred(j)
            return max(copy + h + dd, kern + k)
        if policy == W.MBF:                         # L831: avoid co-locating bandwidth-bound kernels
            sh = sd = shbm = ssm = 0
            for i in res + [j]:
                h, k, dd, _ = self.pred(i)
                fresh = i is j
                if fresh or i.phase <= H2D:
                    sh += h
                if fresh or i.phase <= D2H:
                    sd += dd
                if fresh or i.phase <= KL:
                    hb = min(k, ceil_div(i.hbm_bytes, PRIOR_HBM_BYTES_PER_NS))
                    shbm += hb
                    ssm += k - hb
            return max(sh, sd, shbm, ssm)
        raise ValueError(policy)

    def select_device(self, policy: int, j: Job, admissible: List[Device]) -> Tuple[Device, int]:
        if policy == W.GRR:                          # L683
            for k in range(self.G):
                g = (self.grr_cursor + k) % self.G
                if any(d.gid == g for d in admissible):
                    self.grr_cursor = (g + 1) % self.G
                    return self.devices[g], 0
            raise AssertionError("no admissible device")
        if policy == W.GWTMIN:                       # L689: min load/weight, cross-multiplied
            best = None
            for d in admissible:
                if best is None or len(d.resident) * best.weight < len(best.resident) * d.weight:
                    best = d
            return best, len(best.resident)
        best, bs = None, None
        for d in admissible:                         # ties -> lowest GID (L687, R-13)
            s = self.score(policy, j, d)
            if bs is None or s < bs:
                best, bs = d, s
        return best, bs

    # --------------------------------------------------------------- admission
    def admission(self, t: int) -> None:
        """Balancer admission loop (S2; R-9, R-16)."""
        while True:
            elig = []
            for tid, tn in enumerate(self.tenants):
                if tn.pending and tn.inflight < tn.c:
                    j = self.jobs[tn.pending[0]]
                    if j.arrived:
                        elig.append(j)
            adm = [d for d in self.devices if len(d.resident) < self.M]
            if not elig or not adm:
                return
            order = self.admission_sorted(elig)
            joint = self.cfg.joint_select and self.cfg.balancer in (W.DTF, W.MBF, W.DYNAMIC)
            if joint:
                cold = [j for j in order if self.effective_policy(j) == W.GMIN]
                if cold:
                    j = cold[0]
                    pol = W.GMIN
                    d, s = self.select_device(pol, j, adm)
                else:
                    best = None
                    for j_ in order:                 # admission rank, then GID
                        pol_ = self.effective_policy(j_)
                        for d_ in adm:
                            s_ = self.score(pol_, j_, d_)
                            if best is None or s_ < best[0]:
                                best = (s_, j_, d_, pol_)
                    s, j, d, pol = best
            else:
                j = order[0]
                pol = self.effective_policy(j)
                d, s = self.select_device(pol, j, adm)
            self.place(t, j, d, pol, s)

    def place(self, t, j: Job, d: Device, pol: int, score: int) -> None:
        tn = self.tenants[j.tenant]
        assert tn.pending[0] == j.id
        tn.pending.pop(0)
        tn.inflight += 1
        j.placed, j.gid, j.t_place = True, d.gid, t
        j.place_order = self.place_counter
        self.place_counter += 1
        d.resident.append(j.id)
        self.rec(t, "PLACE", d.gid, None, None, j.tenant, j.seq, j.id, pol, score)

    # ----------------------------------------------------------------- dispatch
    def wake(self, t, d: Device, j: Job) -> None:
        j.woken = True
        d.fifo[j.phase].append(j.id)
        d.woken_unfinished += 1
        self.rec(t, "WAKE", d.gid, j.phase, None, j.tenant, j.seq, j.id)

    def dispatch(self, t, d: Device) -> None:
        """Device dispatch pass (S5, R-11): choose which ready phases to wake."""
        cands = [self.jobs[i] for i in d.resident]
        cands = [j for j in cands if j.phase < 3 and not j.woken]
        free = self.A - d.woken_unfinished
        pol = self.cfg.device_policy
        if cands and free > 0:
            if pol == W.FIFO:
                for j in sorted(cands, key=lambda j: j.place_order)[:free]:
                    self.wake(t, d, j)
            elif pol == W.LAS:                        # L693: phase-blind, least service first
                for j in self.las_sorted(cands)[:free]:
                    self.wake(t, d, j)
            elif pol == W.PS:                         # L819
                by = {x: self.las_sorted([j for j in cands if j.phase == x]) for x in (H2D, KL, D2H)}
                active = [0, 0, 0]
                for x in (H2D, KL, D2H):
                    active[x] = len(d.fifo[x]) + sum(1 for b in d.busy[x] if b is not None)
                # (i) diversity: one woken op per phase, KL first
                if active[KL] == 0 and by[KL] and free > 0:
                    self.wake(t, d, by[KL].pop(0))
                    free -= 1
                copies = [x for x in (H2D, D2H) if active[x] == 0 and by[x]]
                if len(copies) == 2 and self.las_key_less(by[D2H][0], by[H2D][0]):
                    copies = [D2H, H2D]               # lower min-key first; exact tie -> H2D
                for x in copies:
                    if free > 0:
                        self.wake(t, d, by[x].pop(0))
                        free -= 1
                # (ii) fill: KL > H2D = D2H
                for j in list(by[KL]):
                    if free > 0:
                        self.wake(t, d, j)
                        free -= 1
                for j in self.las_sorted(by[H2D] + by[D2H]):
                    if free > 0:
                        self.wake(t, d, j)
                        free -= 1
            elif pol == W.TFS:                        # L699, L817 (R-28)
                self.tfs_wake(t, d, cands, free)
            else:
                raise ValueError(pol)
        elif pol == W.TFS:
            self.tfs_wake(t, d, cands, free)         # release bookkeeping even with no budget
        # start pass: free engines / slots take their FIFO heads
        for x in (H2D, KL, D2H):
            for s in range(len(d.busy[x])):
                if d.busy[x][s] is None and d.fifo[x]:
                    j = self.jobs[d.fifo[x].pop(0)]
                    d.busy[x][s] = j.id
                    j.start[x], j.slot[x] = t, s
                    self.rec(t, "START", d.gid, x, s, j.tenant, j.seq, j.id)
                    heapq.heappush(self.done_heap, (t + j.dur[x], d.gid, x, s, j.id))

    def tfs_wake(self, t, d: Device, cands: List[Job], free: int) -> None:
        """True Fair-Share: only the awake tenant's ops may be woken (at most one
        backend thread awake, L699).  It stays awake until it has used w_t * S of
        service on this device since it woke, or has nothing to run (work
        conserving, L817); it is released only once its woken ops finished.  The
        next tenant is the one with the least service / weight on this device
        (cumulative, so an overshoot is paid back in later turns, L817)."""
        if d.awake is not None:
            w = self.tenants[d.awake].weight
            mine = [j for j in cands if j.tenant == d.awake]
            if d.woken_unfinished == 0 and (d.awake_used >= w * self.S or not mine):
                d.awake = None
        if d.awake is None:
            best = None
            for tid in sorted({j.tenant for j in cands}):
                if best is None or d.svc.get(tid, 0) * self.tenants[best].weight < \
                        d.svc.get(best, 0) * self.tenants[tid].weight:
                    best = tid
            if best is not None:
                d.awake, d.awake_used = best, 0
        if d.awake is None or d.awake_used >= self.tenants[d.awake].weight * self.S:
            return
        for j in sorted((j for j in cands if j.tenant == d.awake), key=lambda j: j.place_order):
            if free <= 0:
                break
            self.wake(t, d, j)
            free -= 1

    # -------------------------------------------------------------- completions
    def complete(self, t, gid, x, s, jid) -> None:
        d, j = self.devices[gid], self.jobs[jid]
        tn = self.tenants[j.tenant]
        assert d.busy[x][s] == jid
        d.busy[x][s] = None
        d.woken_unfinished -= 1
        j.done[x] = t
        j.phase += 1
        j.woken = False
        tn.gs_acc += t - max(j.start[x], self.epoch_start)
        d.svc[j.tenant] = d.svc.get(j.tenant, 0) + (t - j.start[x])
        if d.awake == j.tenant:
            d.awake_used += t - j.start[x]
        self.rec(t, "DONE", gid, x, s, j.tenant, j.seq, jid, t - j.start[x])
        if x == D2H:
            j.t_jobdone = t
            self.jobs_done += 1
            self.rec(t, "JOB_DONE", gid, None, None, j.tenant, j.seq, jid, t - j.arrival)
            self.feedback(t, j)
            d.resident.remove(jid)
            tn.inflight -= 1

    def feedback(self, t, j: Job) -> None:
        """Request Monitor -> Feedback Engine -> SFT (L671-673, L311; R-14)."""
        smp = [j.done[x] - j.start[x] for x in (H2D, KL, D2H)]
        span = t - j.t_place
        util = smp[KL] * 65536 // span if span > 0 else 0
        e = self.sft.setdefault((j.tenant, j.spec.kclass), SFTEntry())
        if e.count == 0:
            e.h2d, e.kl, e.d2h, e.util = smp[0], smp[1], smp[2], util
        else:                                         # same k = 4/5 as Eq. (1)
            e.h2d = (4 * smp[0] + e.h2d) // 5
            e.kl = (4 * smp[1] + e.kl) // 5
            e.d2h = (4 * smp[2] + e.d2h) // 5
            e.util = (4 * util + e.util) // 5
        e.count += 1
        self.rec(t, "FEEDBACK", j.gid, None, None, j.tenant, j.seq, j.id, e.h2d + e.d2h, e.kl)

    def epoch(self, t) -> None:
        """Close epoch [t-Q, t): GS_n per tenant, then Eq. (1) (L695; R-4, R-6)."""
        inprog = [0] * len(self.tenants)
        for d in self.devices:
            for x in (H2D, KL, D2H):
                for jid in d.busy[x]:
                    if jid is not None:
                        j = self.jobs[jid]
                        inprog[j.tenant] += t - max(j.start[x], self.epoch_start)
        for tid, tn in enumerate(self.tenants):
            gs = tn.gs_acc + inprog[tid]
            old = tn.cgs
            tn.cgs = (4 * (gs << 16) + old) // 5
            tn.gs_acc = 0
            if gs > 0 or old > 0:
                self.rec(t, "EPOCH", None, None, None, tid, None, None, gs, tn.cgs)
        self.epoch_start = t
        self.next_epoch = t + self.Q

    # --------------------------------------------------------------- main loop
    def process(self, t: int) -> None:
        first = True
        while True:
            batch = []
            while self.done_heap and self.done_heap[0][0] == t:
                batch.append(heapq.heappop(self.done_heap))
            batch.sort()                              # (GID, engine, slot, job)  R-10
            for _, gid, x, s, jid in batch:
                self.complete(t, gid, x, s, jid)
            if first:
                if self.next_epoch == t:
                    self.epoch(t)
                while (self.next_arrival < len(self.arrival_order)
                       and self.jobs[self.arrival_order[self.next_arrival]].arrival == t):
                    j = self.jobs[self.arrival_order[self.next_arrival]]
                    j.arrived = True
                    self.next_arrival += 1
                    self.rec(t, "ARRIVE", None, None, None, j.tenant, j.seq, j.id, j.prio)
                first = False
            self.admission(t)
            for d in self.devices:
                self.dispatch(t, d)
            if not (self.done_heap and self.done_heap[0][0] == t):
                return

    def run(self) -> "Oracle":
        while self.jobs_done < len(self.jobs):
            cand = []
            if self.done_heap:
                cand.append(self.done_heap[0][0])
            if self.next_arrival < len(self.arrival_order):
                cand.append(self.jobs[self.arrival_order[self.next_arrival]].arrival)
            if not cand:
                raise RuntimeError("scheduler deadlock: unfinished jobs but no pending event")
            cand.append(self.next_epoch)
            self.process(min(cand))
        return self


def run_oracle(wl: W.Workload) -> Oracle:
    return Oracle(wl).run()
