"""Invariant checker for decision traces (oracle or GPU path, any timing mode).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Checks the invariants of SURVEY.md §8(c) on a canonical trace:
  I1  no job lost or duplicated: exactly one ARRIVE, PLACE, JOB_DONE and one
      WAKE/START/DONE per phase, in the order H2D < KL < D2H, on one GID.
  I2  LAS ordering: every LAS admission (when LAS admission is on and joint
      selection is off) places a job of minimal weighted key among the
      eligible ones; every LAS-policy wake takes a minimal-key candidate of its
      device at that moment (reading R-7); every PS wake takes a
      minimal-key candidate among the device's candidates of the same phase
      (reading R-11).
  I3  resource exclusivity: <= 1 op per copy engine, <= P KL ops per device,
      <= A woken-unfinished ops, <= M resident jobs, <= c_t in-flight per tenant.
  I4  per-tenant order: a tenant's jobs are admitted in
      submission order; with one server thread (c_t = 1) each phase of job s+1
      starts after job s's.  Jobs admitted concurrently (c_t > 1, the finite
      server threads of L879) are independent requests (reading R-27).
  I5  work conservation at the end of every timestamp: no engine idles while
      an op is woken for it; no candidate stays unwoken while budget remains
      (TFS: no device sits with candidates and nothing woken).
  I7  TFS: the woken-unfinished ops of a device belong to at
      most one tenant at any time.
"""
from __future__ import annotations

import functools
from dataclasses import dataclass
from typing import Dict, List, Optional, Tuple

import strings_workload as W

ENG = {"H2D": 0, "KL": 1, "D2H": 2}


@dataclass
class Rec:
    idx: int
    t: int
    kind: str
    gid: Optional[int]
    eng: Optional[int]
    slot: Optional[int]
    tenant: Optional[int]
    seq: Optional[int]
    job: Optional[int]
    a1: int
    a2: int


def _opt(s: str) -> Optional[int]:
    return None if s == "-" else int(s)


def parse(lines: List[str]) -> List[Rec]:
    out = []
    for i, ln in enumerate(lines):
        f = ln.split()
        if len(f) != 10:
            raise ValueError(f"bad trace line {i}: {ln!r}")
        out.append(Rec(i, int(f[0]), f[1], _opt(f[2]), None if f[3] == "-" else ENG[f[3]],
                       _opt(f[4]), _opt(f[5]), _opt(f[6]), _opt(f[7]), int(f[8]), int(f[9])))
    return out


def check(lines: List[str], wl: W.Workload) -> List[str]:
    cfg = wl.config.resolved()
    G, P, A, M = cfg.num_gpus, cfg.partitions, cfg.awake_budget, cfg.admit_cap
    recs = parse(lines)
    errs: List[str] = []
    J = len(wl.jobs)
    ten_of = [j.tenant for j in wl.jobs]
    seq_of, cnt = [], {}
    for j in wl.jobs:
        seq_of.append(cnt.get(j.tenant, 0))
        cnt[j.tenant] = seq_of[-1] + 1

    # ---- I1: per-job record shape and order ---------------------------------
    per_job: Dict[int, List[Rec]] = {i: [] for i in range(J)}
    last_t = None
    for r in recs:
        if last_t is not None and r.t < last_t:
            errs.append(f"I1 time goes backwards at record {r.idx}")
        last_t = r.t
        if r.job is not None:
            if not (0 <= r.job < J):
                errs.append(f"I1 unknown job {r.job}")
                continue
            if r.tenant != ten_of[r.job] or r.seq != seq_of[r.job]:
                errs.append(f"I1 job {r.job} tenant/seq mismatch at record {r.idx}")
            per_job[r.job].append(r)
    expect = ["ARRIVE", "PLACE"]
    for e in ("H2D", "KL", "D2H"):
        expect += [f"WAKE:{e}", f"START:{e}", f"DONE:{e}"]
    expect += ["JOB_DONE", "FEEDBACK"]
    for jid, rs in per_job.items():
        got = [r.kind + (f":{'H2D KL D2H'.split()[r.eng]}" if r.eng is not None else "") for r in rs]
        if got != expect:
            errs.append(f"I1 job {jid} record sequence {got}")
            continue
        gids = {r.gid for r in rs if r.kind not in ("ARRIVE",)}
        if len(gids) != 1:
            errs.append(f"I1 job {jid} on several GIDs {gids}")

    # ---- replay for I2..I5 ----------------------------------------------------
    busy = [[[None], [None] * P, [None]] for _ in range(G)]
    fifo = [[[], [], []] for _ in range(G)]
    woken_unf = [0] * G
    resident: List[List[int]] = [[] for _ in range(G)]
    inflight = [0] * len(wl.tenants)
    phase = [0] * J              # phases done
    woken = [False] * J
    arrived = [False] * J
    placed = [False] * J
    prio = [0] * J
    cgs = [0] * len(wl.tenants)
    pending: Dict[int, List[int]] = {t: [] for t in range(len(wl.tenants))}
    for i, j in enumerate(wl.jobs):
        pending[j.tenant].append(i)
    last_start: Dict[Tuple[int, int], int] = {}
    last_place: Dict[int, int] = {}
    joint = cfg.joint_select and cfg.balancer in (W.DTF, W.MBF, W.DYNAMIC)

    def las_cmp(a, b):
        lhs, rhs = cgs[ten_of[a]] * prio[b], cgs[ten_of[b]] * prio[a]
        if lhs != rhs:
            return -1 if lhs < rhs else 1
        return -1 if (ten_of[a], seq_of[a]) < (ten_of[b], seq_of[b]) else 1

    def candidates(g):
        return [i for i in resident[g] if phase[i] < 3 and not woken[i]]

    def end_of_timestamp(t, woken_now):
        for g in range(G):
            for x in range(3):
                if fifo[g][x] and any(b is None for b in busy[g][x]):
                    errs.append(f"I5 t={t} gid={g} engine {x} idle with woken op")
            c = candidates(g)
            if cfg.device_policy == W.TFS:
                if c and woken_unf[g] == 0:
                    errs.append(f"I5 t={t} gid={g} TFS device idle with {len(c)} candidates")
            elif c and woken_unf[g] < A:
                errs.append(f"I5 t={t} gid={g} {len(c)} candidates unwoken with budget {A - woken_unf[g]}")


    cur_t = None
    woken_now: Dict[int, List[int]] = {}
    epoch_seen_t = None
    for r in recs:
        if cur_t is not None and r.t != cur_t:
            end_of_timestamp(cur_t, woken_now)
            woken_now = {}
        cur_t = r.t
        k = r.kind
        if k == "EPOCH":
            if epoch_seen_t != r.t:
                cgs = [0] * len(wl.tenants)      # tenants without a record have CGS 0
                epoch_seen_t = r.t
            cgs[r.tenant] = r.a2
        elif k == "ARRIVE":
            arrived[r.job] = True
            prio[r.job] = r.a1
        elif k == "PLACE":
            j, g, tn = r.job, r.gid, r.tenant
            if not arrived[j]:
                errs.append(f"I1 job {j} placed before arrival")
            if pending[tn] and pending[tn][0] != j:
                errs.append(f"I4 tenant {tn} placed job {j} before {pending[tn][0]}")
            if cfg.las_admission and not joint:
                elig = [pending[t][0] for t in pending if pending[t] and arrived[pending[t][0]]
                        and inflight[t] < wl.tenants[t].max_inflight]
                for e in elig:
                    if e != j and las_cmp(e, j) < 0:
                        errs.append(f"I2 t={r.t} admitted job {j} before lower-key job {e}")
            if pending[tn] and pending[tn][0] == j:
                pending[tn].pop(0)
            placed[j] = True
            resident[g].append(j)
            inflight[tn] += 1
            if len(resident[g]) > M:
                errs.append(f"I3 gid {g} resident {len(resident[g])} > M={M}")
            if inflight[tn] > wl.tenants[tn].max_inflight:
                errs.append(f"I3 tenant {tn} in-flight {inflight[tn]} > c_t")
        elif k == "WAKE":
            j, g, x = r.job, r.gid, r.eng
            if phase[j] != x or woken[j]:
                errs.append(f"I1 job {j} woken for phase {x} out of order")
            if cfg.device_policy == W.LAS:
                # a LAS pass wakes candidates in key order: each woken job has the
                # minimal key among the device's candidates at that moment (exact
                # per pass, even when one timestamp holds several passes)
                for u in candidates(g):
                    if u != j and las_cmp(u, j) < 0:
                        errs.append(f"I2 t={r.t} gid={g} LAS woke job {j} before lower-key job {u}")
            if cfg.device_policy == W.PS:
                # PS (R-11) chooses *which phases* to wake, but
                # within a phase it always takes the minimal-key candidate
                # (diversity step and fill step alike)
                for u in candidates(g):
                    if u != j and phase[u] == x and las_cmp(u, j) < 0:
                        errs.append(f"I2 t={r.t} gid={g} PS woke job {j} before lower-key job {u} of its phase")
            if cfg.device_policy == W.TFS:
                others = {ten_of[i] for i in resident[g] if woken[i]} - {ten_of[j]}
                if others:
                    errs.append(f"I7 t={r.t} gid={g} TFS woke tenant {ten_of[j]} while {others} awake")
            woken[j] = True
            fifo[g][x].append(j)
            woken_unf[g] += 1
            woken_now.setdefault(g, []).append(j)
            if woken_unf[g] > A:
                errs.append(f"I3 gid {g} woken-unfinished {woken_unf[g]} > A={A}")
        elif k == "START":
            j, g, x, s = r.job, r.gid, r.eng, r.slot
            if s is None or s >= len(busy[g][x]):
                errs.append(f"I3 bad slot {s} for engine {x}")
                continue
            if busy[g][x][s] is not None:
                errs.append(f"I3 t={r.t} gid {g} engine {x} slot {s} started while busy")
            if not fifo[g][x] or fifo[g][x][0] != j:
                errs.append(f"I3 t={r.t} gid {g} engine {x} started job {j} out of FIFO order")
            if j in fifo[g][x]:
                fifo[g][x].remove(j)
            busy[g][x][s] = j
            key = (ten_of[j], x)
            if (wl.tenants[ten_of[j]].max_inflight == 1 and key in last_start
                    and seq_of[last_start[key]] > seq_of[j]):
                errs.append(f"I4 tenant {ten_of[j]} engine {x} job {j} started after a later job")
            last_start[key] = j
        elif k == "DONE":
            j, g, x, s = r.job, r.gid, r.eng, r.slot
            if s is None or s >= len(busy[g][x]) or busy[g][x][s] != j:
                errs.append(f"I3 t={r.t} DONE of job {j} not running on gid {g} engine {x} slot {s}")
            else:
                busy[g][x][s] = None
            phase[j] += 1
            woken[j] = False
            woken_unf[g] -= 1
        elif k == "JOB_DONE":
            j, g = r.job, r.gid
            if j in resident[g]:
                resident[g].remove(j)
            inflight[ten_of[j]] -= 1
    if cur_t is not None:
        end_of_timestamp(cur_t, woken_now)
    return errs
