"""Pins for the scheduler oracle (oracle/des.py) -- no GPU.

Each test ties the DES to something other than itself: a rule the paper states
(as a hand-worked case), a textbook closed form, a brute-force optimum or a
classical bound.
"""
import itertools
import math

import numpy as np
import pytest

import strings_workload as W
from oracle import bruteforce, invariants
from oracle.des import D2H, H2D, KL, Oracle, SFTEntry, run_oracle


def kl_only_job(t, kl_ns, arrival=0, prio=0):
    """A job whose H2D/D2H move zero bytes and whose KL takes kl_ns (VSCALE n=0)."""
    return W.JobSpec(tenant=t, kclass=W.VSCALE, n=0, arrival_ns=arrival, priority=prio,
                     inj_h2d_ns=0, inj_kl_ns=kl_ns, inj_d2h_ns=0)


def wakes(o, t=None):
    return [ln.split() for ln in o.trace if ln.split()[1] == "WAKE" and (t is None or int(ln.split()[0]) == t)]


# ------------------------------------------------------------------ PS rule
def ps_state(A, jobs, policy=W.PS):
    """Hand-built device state: jobs = [(phase, cgs)], one tenant per job,
    all resident on GID 0, nothing woken yet.  Returns (oracle, WAKE list)."""
    cfg = W.SystemConfig(num_gpus=1, device_policy=policy, partitions=3, awake_budget=A, admit_cap=64)
    tenants = [W.TenantSpec() for _ in jobs]
    specs = [kl_only_job(i, 100) for i in range(len(jobs))]
    o = Oracle(W.Workload("ps", cfg, tenants, specs))
    d = o.devices[0]
    for i, (ph, cgs) in enumerate(jobs):
        j = o.jobs[i]
        o.tenants[i].cgs = cgs
        o.tenants[i].pending.clear()
        j.arrived = j.placed = True
        j.gid, j.phase, j.place_order = 0, ph, i
        d.resident.append(i)
    o.dispatch(0, d)
    return o, [(int(w[7]), w[3]) for w in wakes(o)]


def test_ps_one_of_each_phase():
    # {>=1 KL, H2D, D2H candidate; A=3} -> one of each
    _, w = ps_state(3, [(KL, 5), (KL, 6), (H2D, 1), (D2H, 2)])
    assert sorted(p for _, p in w) == ["D2H", "H2D", "KL"]
    assert (0, "KL") in w                       # the min-key KL


def test_ps_missing_phase_fills_by_priority():
    # {>=2 KL, >=1 D2H, no H2D; A=3} -> 2 KL + 1 D2H
    _, w = ps_state(3, [(KL, 5), (KL, 6), (KL, 7), (D2H, 1)])
    assert sorted(p for _, p in w) == ["D2H", "KL", "KL"]
    assert {j for j, p in w if p == "KL"} == {0, 1}


def test_ps_budget_one_prefers_kl():
    # {KL, H2D, D2H; A=1} -> KL (KL > H2D = D2H)
    _, w = ps_state(1, [(H2D, 0), (D2H, 0), (KL, 9)])
    assert w == [(2, "KL")]


def test_ps_copies_ordered_by_key():
    # {H2D key 5, D2H key 3, no KL; A=1} -> D2H ; equal keys -> H2D
    _, w = ps_state(1, [(H2D, 5), (D2H, 3)])
    assert w == [(1, "D2H")]
    _, w = ps_state(1, [(D2H, 4), (H2D, 4)])
    assert w == [(1, "H2D")]


def test_ps_differs_from_las():
    # three lowest keys are H2D candidates, one KL candidate, no D2H; A=3
    state = [(H2D, 1), (H2D, 2), (H2D, 3), (KL, 9)]
    _, las = ps_state(3, state, policy=W.LAS)
    _, ps = ps_state(3, state, policy=W.PS)
    assert sorted(las) == [(0, "H2D"), (1, "H2D"), (2, "H2D")]           # phase-blind by key
    assert sorted(ps) == [(0, "H2D"), (1, "H2D"), (3, "KL")]             # diversity then fill


def test_fifo_wakes_in_placement_order():
    _, w = ps_state(2, [(KL, 9), (H2D, 1), (D2H, 0)], policy=W.FIFO)
    assert w == [(0, "KL"), (1, "H2D")]


# ------------------------------------------------------------ balancer rules
def placements(o):
    return [int(ln.split()[2]) for ln in o.trace if ln.split()[1] == "PLACE"]


def test_grr_round_robin():
    cfg = W.SystemConfig(num_gpus=3, balancer=W.GRR, admit_cap=100)
    wl = W.Workload("grr", cfg, [W.TenantSpec(max_inflight=100)],
                    [kl_only_job(0, 1000 * (i + 1)) for i in range(7)])
    assert placements(run_oracle(wl)) == [0, 1, 2, 0, 1, 2, 0]


def test_gmin_least_loaded_and_lowest_gid_ties():
    cfg = W.SystemConfig(num_gpus=3, balancer=W.GMIN, admit_cap=100)
    # long job first, then three that arrive after shorter ones finished
    jobs = [kl_only_job(0, 10_000), kl_only_job(1, 100), kl_only_job(2, 100),
            kl_only_job(3, 50, arrival=1000), kl_only_job(4, 50, arrival=1000)]
    o = run_oracle(W.Workload("gmin", cfg, [W.TenantSpec() for _ in range(5)], jobs))
    # t=0: 0->0, 1->1, 2->2 ; t=1000: GIDs 1,2 are empty, GID 0 holds one -> 1 then 2
    assert placements(o) == [0, 1, 2, 1, 2]


def test_gwtmin_equals_gmin_with_equal_weights_and_gmin_equals_grr_for_equal_jobs():
    base = [kl_only_job(t % 4, 500, arrival=(t // 4) * 100) for t in range(12)]
    out = {}
    for pol in (W.GRR, W.GMIN, W.GWTMIN):
        cfg = W.SystemConfig(num_gpus=3, balancer=pol, admit_cap=100)
        wl = W.Workload("eq", cfg, [W.TenantSpec(max_inflight=8) for _ in range(4)],
                        [W.JobSpec(**vars(j)) for j in base])
        out[pol] = placements(run_oracle(wl))
    assert out[W.GMIN] == out[W.GWTMIN] == out[W.GRR]


def seeded_oracle(policy, G, job_preds, joint=0):
    """All jobs arrived at t=0, one tenant per job with an SFT sample equal to
    job_preds[i] = (h2d, kl, d2h); M = c_t = infinity.  Runs one admission pass
    (nothing has started) and returns (oracle, placement list)."""
    cfg = W.SystemConfig(num_gpus=G, balancer=policy, admit_cap=10 ** 6, joint_select=joint)
    specs = []
    for i, (h, k, d) in enumerate(job_preds):
        specs.append(W.JobSpec(tenant=i, kclass=W.GEMM, m=128, n=256, k=64, inj_h2d_ns=h,
                               inj_kl_ns=k, inj_d2h_ns=d))
    o = Oracle(W.Workload("seed", cfg, [W.TenantSpec() for _ in job_preds], specs))
    for i, (h, k, d) in enumerate(job_preds):
        o.sft[(i, W.GEMM)] = SFTEntry(count=1, h2d=h, kl=k, d2h=d, util=0)
        o.jobs[i].arrived = True
    o.admission(0)
    pl = [0] * len(job_preds)
    for ln in o.trace:
        f = ln.split()
        if f[1] == "PLACE":
            pl[int(f[7])] = int(f[2])
    return o, pl


@pytest.mark.parametrize("seed", range(40))
def test_rtf_is_list_scheduling_within_graham_bound(seed):
    # RTF with all jobs placed before anything runs = greedy least-loaded list
    # scheduling on predicted runtime: max load <= (2 - 1/G) * OPT (Graham 1966)
    rng = np.random.default_rng(seed)
    G = int(rng.integers(2, 4))
    J = int(rng.integers(2, 8))
    p = [int(x) for x in rng.integers(1, 100, J)]
    _, pl = seeded_oracle(W.RTF, G, [(0, x, 0) for x in p])
    load = bruteforce.vector_load([[x] for x in p], pl, G)
    opt, _ = bruteforce.optimal_vector_load([[x] for x in p], G)
    assert load * G <= (2 * G - 1) * opt
    # LPT order (tenant 0 largest) tightens it to (4/3 - 1/(3G)) * OPT
    q = sorted(p, reverse=True)
    _, pl2 = seeded_oracle(W.RTF, G, [(0, x, 0) for x in q])
    load2 = bruteforce.vector_load([[x] for x in q], pl2, G)
    assert 3 * G * load2 <= (4 * G - 1) * opt


def mbf_vectors(preds, hbm_parts):
    out = []
    for (h, k, d), hb in zip(preds, hbm_parts):
        hb = min(k, hb)
        out.append([h, d, hb, k - hb])
    return out


def test_mbf_designed_case_reaches_optimum():
    # config-1 shape: 2 VSCALE-like (HBM-bound) + 2 GEMM-like (SM-bound), G=2.
    # GEMM 128x256x64 has 2*(128*64+64*256)+4*128*256 = 180224 B -> 31 ns of HBM.
    preds = [(80_000, 1_400, 80_000), (80_000, 1_400, 80_000), (5_000, 97_000, 5_000), (5_000, 97_000, 5_000)]
    for joint in (0, 1):
        o, pl = seeded_oracle(W.MBF, 2, preds, joint=joint)
        hb = [min(k, math.ceil(o.jobs[i].hbm_bytes / 6000)) for i, (_, k, _) in enumerate(preds)]
        vec = mbf_vectors(preds, hb)
        opt, _ = bruteforce.optimal_vector_load(vec, 2)
        assert bruteforce.vector_load(vec, pl, 2) == opt
        assert pl[0] != pl[1] and pl[2] != pl[3]        # one of each class per GPU


@pytest.mark.parametrize("seed", range(40))
@pytest.mark.parametrize("policy", [W.MBF, W.DTF])
def test_vector_greedy_within_d_plus_one_of_optimum(seed, policy):
    rng = np.random.default_rng(1000 + seed)
    G = int(rng.integers(2, 4))
    J = int(rng.integers(2, 7))
    preds = [tuple(int(x) for x in rng.integers(0, 1000, 3)) for _ in range(J)]
    for joint in (0, 1):
        o, pl = seeded_oracle(policy, G, preds, joint=joint)
        if policy == W.MBF:
            hb = [math.ceil(o.jobs[i].hbm_bytes / 6000) for i in range(J)]
            vec = mbf_vectors(preds, hb)
        else:
            vec = [[h + d, k] for (h, k, d) in preds]
        dim = len(vec[0])
        opt, _ = bruteforce.optimal_vector_load(vec, G)
        assert bruteforce.vector_load(vec, pl, G) <= (dim + 1) * opt


def test_mbf_spreads_bandwidth_bound_jobs():
    # n_b identical bandwidth-bound jobs on G empty devices: none gets > ceil(n_b/G)
    for G in (2, 3):
        for nb in range(1, 8):
            _, pl = seeded_oracle(W.MBF, G, [(10, 1000, 10)] * nb)
            counts = [pl.count(g) for g in range(G)]
            assert max(counts) <= -(-nb // G)


def test_dynamic_uses_gmin_until_feedback():
    wl = W.config_c5()
    o = run_oracle(wl)
    pol = {}
    for ln in o.trace:
        f = ln.split()
        if f[1] == "PLACE":
            pol.setdefault(int(f[5]), []).append(int(f[8]))
    # every tenant's first job is cold -> GMin; later jobs of a known class -> MBF
    assert all(v[0] == W.GMIN for v in pol.values())
    assert any(W.MBF in v for v in pol.values())


# ------------------------------------------------------------------ Eq. (1)
def test_eq1_worked_decay():
    # Tenant 0: one 10 ms KL job from t=0; Q = 10 ms.  Tenant 1 keeps the
    # system alive until 35 ms.  GS = [10 ms, 0, 0] -> CGS = 8, 1.6, 0.32 ms.
    cfg = W.SystemConfig(num_gpus=1, device_policy=W.FIFO, partitions=2, quantum_ns=10_000_000)
    wl = W.Workload("eq1", cfg, [W.TenantSpec(), W.TenantSpec()],
                    [kl_only_job(0, 10_000_000), kl_only_job(1, 1, arrival=35_000_000)])
    o = run_oracle(wl)
    ep = [(int(f[0]), int(f[8]), int(f[9])) for f in (ln.split() for ln in o.trace)
          if f[1] == "EPOCH" and f[5] == "0"]
    assert [t for t, _, _ in ep[:3]] == [10_000_000, 20_000_000, 30_000_000]
    assert [g for _, g, _ in ep[:3]] == [10_000_000, 0, 0]
    for (_, _, cgs), ms in zip(ep[:3], (8.0, 1.6, 0.32)):
        assert abs(cgs / 65536 - ms * 1e6) <= 1.0            # within 1 ns (Q16 floor)


def test_eq1_constant_service_converges_geometrically():
    # GS = g every epoch -> CGS_n = g * (1 - 0.2^n); integer floor error < n ulps(Q16)
    g = 1000
    cfg = W.SystemConfig(num_gpus=1, device_policy=W.FIFO, quantum_ns=g)
    o = run_oracle(W.Workload("c", cfg, [W.TenantSpec()], [kl_only_job(0, 12 * g)]))
    cg = [int(f[9]) for f in (ln.split() for ln in o.trace) if f[1] == "EPOCH"]
    assert len(cg) == 12                     # one per epoch the 12g op spans (in-progress service)
    for n, c in enumerate(cg, start=1):
        exact = g * (1 - 0.2 ** n) * 65536
        assert exact - n <= c <= exact + 1e-6


# ------------------------------------------------------------------- M/M/1
@pytest.mark.slow
@pytest.mark.parametrize("policy", [W.FIFO, W.LAS, W.PS])
def test_mm1_mean_response_time(policy):
    # G=P=A=1, zero-byte copies, Poisson arrivals (Eq. 4), exponential KL
    # sizes, size-blind work-conserving order => E[T] = 1/(mu - lambda).
    mean_s, rho, T, per = 10_000.0, 0.5, 8, 25_000          # 2*10^5 jobs
    rng = W.SplitMix64(2024 + policy)
    jobs = []
    for t in range(T):
        now = 0
        for _ in range(per):
            now += W.exp_interarrival_ns(rng, mean_s * T / rho)
            jobs.append(kl_only_job(t, max(1, W.exp_interarrival_ns(rng, mean_s)), arrival=now))
    jobs.sort(key=lambda j: (j.arrival_ns, j.tenant))
    cfg = W.SystemConfig(num_gpus=1, partitions=1, awake_budget=1, admit_cap=10 ** 6,
                         device_policy=policy, quantum_ns=50_000)
    o = run_oracle(W.Workload("mm1", cfg, [W.TenantSpec(max_inflight=10 ** 6) for _ in range(T)], jobs))
    resp = np.array([j.done[KL] - j.arrival for j in o.jobs], dtype=np.float64)
    svc = np.array([j.dur[KL] for j in o.jobs], dtype=np.float64)
    mu = 1.0 / svc.mean()
    lam = len(jobs) / max(j.arrival for j in o.jobs)
    want = 1.0 / (mu - lam)
    assert abs(resp.mean() / want - 1.0) < 0.03


# ---------------------------------------------------------- roofline (I6)
def device_lower_bound(o, g):
    js = [j for j in o.jobs if j.gid == g]
    if not js:
        return 0
    chain = {}
    for j in js:
        chain[j.tenant] = chain.get(j.tenant, 0) + sum(j.dur)
    return max(sum(j.dur[H2D] for j in js), sum(j.dur[D2H] for j in js),
               -(-sum(j.dur[KL] for j in js) // o.P),
               max(-(-v // o.tenants[t].c) for t, v in chain.items()))


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C5"])
def test_span_respects_roofline_lower_bound(name):
    o = run_oracle(W.CONFIGS[name]())
    for g in range(o.G):
        js = [j for j in o.jobs if j.gid == g]
        if js:
            span = max(j.t_jobdone for j in js) - min(j.start[H2D] for j in js)
            assert span >= device_lower_bound(o, g)


def test_roofline_equality_for_h2d_only_stream():
    cfg = W.SystemConfig(num_gpus=1, awake_budget=2, admit_cap=4, device_policy=W.PS)
    jobs = [W.JobSpec(tenant=0, kclass=W.VSCALE, n=0, inj_h2d_ns=1000 + 7 * i) for i in range(20)]
    o = run_oracle(W.Workload("h2d", cfg, [W.TenantSpec(max_inflight=10 ** 6)], jobs))
    span = max(j.t_jobdone for j in o.jobs)
    assert span == sum(j.dur[H2D] for j in o.jobs)        # the H2D engine never idles


# -------------------------------------------------------------- invariants
@pytest.mark.parametrize("name", list(W.CONFIGS))
def test_configs_satisfy_invariants(name):
    wl = W.CONFIGS[name]()
    o = run_oracle(wl)
    assert invariants.check(o.trace, wl) == []
    assert sum(1 for ln in o.trace if " JOB_DONE " in ln) == len(wl.jobs)


@pytest.mark.parametrize("seed", range(200))
def test_random_workloads_satisfy_invariants(seed):
    wl = W.random_workload(seed)
    o = run_oracle(wl)
    assert invariants.check(o.trace, wl) == []


def test_invariant_checker_catches_mutations():
    wl = W.config_c1()
    tr = run_oracle(wl).trace
    assert invariants.check(tr, wl) == []
    start = next(i for i, l in enumerate(tr) if " START " in l)
    done = next(i for i, l in enumerate(tr) if " JOB_DONE " in l)
    place = [i for i, l in enumerate(tr) if " PLACE " in l]
    mutants = {
        "drop": tr[:start] + tr[start + 1:],
        "dup": tr[:start + 1] + [tr[start]] + tr[start + 1:],
        "lost_job": tr[:done] + tr[done + 2:],
        "wrong_gid": [(" ".join(f[:2] + [str(1 - int(f[2]))] + f[3:]) if i == start else l)
                      for i, (l, f) in enumerate((l, l.split()) for l in tr)],
    }
    for name, m in mutants.items():
        if m is not None:
            assert invariants.check(m, wl), name


# --------------------------------------------------------------------- TFS
def _tfs_shares(policy, weights, sizes=(1_000_000, 50_000), horizon=40_000_000, slice_ns=500_000):
    """Two tenants saturating one device with KL-only jobs of different sizes;
    service each tenant received up to the time the first one runs dry."""
    cfg = W.SystemConfig(num_gpus=1, partitions=1, device_policy=policy, admit_cap=10 ** 6,
                         tfs_slice_ns=slice_ns)
    jobs = []
    counts = [horizon // sizes[0], horizon // sizes[1]]
    for t in (0, 1):
        jobs += [kl_only_job(t, sizes[t]) for _ in range(counts[t])]
    o = run_oracle(W.Workload("tfs", cfg, [W.TenantSpec(weight=w, max_inflight=10 ** 6) for w in weights], jobs))
    end = min(max(j.done[KL] for j in o.jobs if j.tenant == t) for t in (0, 1))
    svc = [sum(max(0, min(j.done[KL], end) - j.start[KL]) for j in o.jobs if j.tenant == t) for t in (0, 1)]
    return svc, o


def test_tfs_equal_weights_fair_share():
    # proportionate share per tenant by weight under high load
    from oracle import metrics
    svc, o = _tfs_shares(W.TFS, (1, 1))
    assert metrics.jain(svc) > 0.99
    fifo, _ = _tfs_shares(W.FIFO, (1, 1))
    assert metrics.jain(fifo) < metrics.jain(svc)          # FIFO is not fair-share


def test_tfs_weights_give_proportional_shares():
    # long jobs overshoot the slice non-preemptively; the service history pays it
    # back, so with jobs well below a slice the shares converge to the weights
    svc, _ = _tfs_shares(W.TFS, (2, 1), sizes=(200_000, 50_000))
    assert abs(svc[0] / svc[1] - 2.0) < 0.1
    svc, _ = _tfs_shares(W.TFS, (1, 3), sizes=(200_000, 50_000))
    assert abs(svc[1] / svc[0] - 3.0) < 0.15


def test_tfs_work_conserving_and_single_awake():
    # a lone tenant keeps the device busy (unused shares go to others, L817)
    cfg = W.SystemConfig(num_gpus=1, partitions=1, device_policy=W.TFS, tfs_slice_ns=1000)
    jobs = [kl_only_job(0, 700) for _ in range(10)] + [kl_only_job(1, 300, arrival=20_000)]
    wl = W.Workload("tfs1", cfg, [W.TenantSpec(max_inflight=100), W.TenantSpec()], jobs)
    o = run_oracle(wl)
    assert max(j.done[KL] for j in o.jobs if j.tenant == 0) == 7000      # no idling
    assert invariants.check(o.trace, wl) == []


def test_ps_relaxes_tfs_for_throughput():
    # PS relaxes the one-awake invariant to overlap phases
    wl = W.config_c2(scale=256, jobs_per_tenant=4)
    spans = {}
    for pol in (W.TFS, W.PS):
        wl.config.device_policy = pol
        o = run_oracle(wl)
        spans[pol] = max(j.t_jobdone for j in o.jobs)
    assert spans[W.PS] < spans[W.TFS]


# ------------------------------------------------------- heterogeneous GWtMin
@pytest.mark.parametrize("weights,jobs", [((2, 1, 1), 12), ((3, 1), 8), ((1, 2, 3), 18)])
def test_gwtmin_places_in_proportion_to_device_weights(weights, jobs):
    # weighted minimum load; with identical jobs placed before any
    # completes, the counts end up proportional to the weights (count/w equalised)
    cfg = W.SystemConfig(num_gpus=len(weights), balancer=W.GWTMIN, admit_cap=10 ** 6,
                         device_weights=list(weights))
    wl = W.Workload("gw", cfg, [W.TenantSpec(max_inflight=10 ** 6)], [kl_only_job(0, 10 ** 6) for _ in range(jobs)])
    pl = placements(run_oracle(wl))
    counts = [pl.count(g) for g in range(len(weights))]
    assert counts == [w * jobs // sum(weights) for w in weights]
    # GMin ignores the weights: equal counts
    cfg.balancer = W.GMIN
    pl = placements(run_oracle(wl))
    assert max(pl.count(g) for g in range(len(weights))) - min(pl.count(g) for g in range(len(weights))) <= 1


def test_invariant_checker_catches_ps_within_phase_wake_order():
    # two same-phase WAKEs of one PS pass swapped must be flagged (I2, R-11)
    wl = W.config_c3()
    tr = run_oracle(wl).trace
    assert invariants.check(tr, wl) == []
    for i in range(len(tr) - 1):
        a, b = tr[i].split(), tr[i + 1].split()
        if (a[1] == b[1] == "WAKE" and a[0] == b[0] and a[2] == b[2] and a[3] == b[3]
                and a[5] != b[5]):
            m = tr[:i] + [tr[i + 1], tr[i]] + tr[i + 2:]
            if any(e.startswith("I2") for e in invariants.check(m, wl)):
                return
    pytest.fail("no PS wake-order mutation detected")


def test_invariant_checker_catches_las_wake_order():
    # a LAS device trace with two WAKEs of one pass swapped must be flagged (I2)
    wl = W.config_c3()
    wl.config.device_policy = W.LAS
    tr = run_oracle(wl).trace
    assert invariants.check(tr, wl) == []
    for i in range(len(tr) - 1):
        a, b = tr[i].split(), tr[i + 1].split()
        if a[1] == b[1] == "WAKE" and a[0] == b[0] and a[2] == b[2] and a[5] != b[5]:
            m = tr[:i] + [tr[i + 1], tr[i]] + tr[i + 2:]
            if any(e.startswith("I2") for e in invariants.check(m, wl)):
                return
    pytest.fail("no LAS wake-order mutation detected")


# ------------------------------------------------ invariant checker, check by check
def _relabel(trace, a, b):
    """Swap jobs a and b (same tenant) in every record: their admissions and
    phase starts then happen in the opposite of submission order."""
    out = []
    for ln in trace:
        f = ln.split()
        if f[7] in (str(a), str(b)):
            ja, jb = (a, b) if f[7] == str(a) else (b, a)
            f[7] = str(jb)
            f[6] = str(_relabel.seq[jb])
        out.append(" ".join(f))
    return out


def test_invariant_checker_each_check_fires():
    # every check of oracle/invariants.py must flag a trace that breaks exactly its rule
    # I4: swap two jobs of one tenant (c_t = 1): admitted and started out of order
    wl = W.config_c1(reps=2)
    o = run_oracle(wl)
    t0 = [j for j in o.jobs if j.tenant == 0]
    _relabel.seq = {j.id: j.seq for j in o.jobs}
    errs = invariants.check(_relabel(o.trace, t0[0].id, t0[1].id), wl)
    assert any("placed job" in e and e.startswith("I4") for e in errs)
    assert any("started after a later job" in e for e in errs)
    # I3: the trace of M = 2 checked against M = 1
    wl2 = W.config_c2(scale=256, jobs_per_tenant=2)
    wl2.config.admit_cap = 2
    tr = run_oracle(wl2).trace
    wl2.config.admit_cap = 1
    assert any(e.startswith("I3") and "> M=1" in e for e in invariants.check(tr, wl2))
    # I5 (budget): the trace of A = 1 checked against A = 3
    wl3 = W.config_c3(scale=16)
    wl3.config.awake_budget, wl3.config.admit_cap = 1, 8
    tr = run_oracle(wl3).trace
    wl3.config.awake_budget = 3
    assert any("candidates unwoken with budget" in e for e in invariants.check(tr, wl3))
    # I5 (idle engine): the trace of P = 1 checked against P = 2 (a woken KL waits beside a free slot)
    cfg4 = W.SystemConfig(num_gpus=1, partitions=1, awake_budget=4, admit_cap=8, device_policy=W.PS)
    wl4 = W.Workload("p1", cfg4, [W.TenantSpec() for _ in range(4)],
                     [kl_only_job(t, 10_000) for _ in range(2) for t in range(4)])
    tr = run_oracle(wl4).trace
    wl4.config.partitions = 2
    assert any("idle with woken op" in e for e in invariants.check(tr, wl4))
    # I7 (TFS): a PS trace checked as TFS wakes several tenants at once
    wl5 = W.config_c2(scale=256, jobs_per_tenant=2)
    tr = run_oracle(wl5).trace
    wl5.config.device_policy = W.TFS
    assert any(e.startswith("I7") for e in invariants.check(tr, wl5))
