"""Hand-worked pins for the balancer scores, the SFT, the PS fill step, the
class priors and Eq. (1) of the scheduler oracle (oracle/des.py) -- no GPU.

Every expected value below is a literal worked out by hand from the paper's
rule (PAPER.md line cited) and the reading DESIGN.md fixes for it; none is
produced by running the oracle.  Each pin is aimed at a plausible slip in the
oracle (a sum that should be a max, a dropped term, a wrong EWMA weight, the
wrong start of a span, a tie broken the wrong way); ``test_oracle_mutations``
applies those slips to a copy of the oracle and checks that some pin fails.
"""
import pytest

import strings_workload as W
from oracle import bruteforce
from oracle.des import D2H, H2D, KL, Oracle, SFTEntry, run_oracle


def kl_only(t, kl_ns, arrival=0, h2d_ns=0, d2h_ns=0):
    """A job moving no bytes, with injected phase durations (inputs)."""
    return W.JobSpec(tenant=t, kclass=W.VSCALE, n=0, arrival_ns=arrival,
                     inj_h2d_ns=h2d_ns, inj_kl_ns=kl_ns, inj_d2h_ns=d2h_ns)


def gemm_job(t):
    # GEMM 128x256x64: 2*(128*64) + 2*(64*256) + 4*(128*256) = 180,224 B of
    # compulsory kernel traffic -> ceil(180224/6000) = 31 ns at the nominal HBM rate
    return W.JobSpec(tenant=t, kclass=W.GEMM, m=128, n=256, k=64)


def warm_oracle(policy, G, preds, joint=0, resident=()):
    """One tenant per job (job i = tenant i, all arrived at t=0) whose SFT row
    (tenant i, GEMM) holds preds[i] = (h2d, kl, d2h, util).  Jobs listed in
    ``resident`` as (job, gid, phase) are already on a device, mid-flight.
    Runs one admission pass at t=0 and returns [(job, gid, score)] in PLACE order."""
    cfg = W.SystemConfig(num_gpus=G, balancer=policy, admit_cap=10 ** 6, joint_select=joint)
    specs = [gemm_job(i) for i in range(len(preds))]
    o = Oracle(W.Workload("pin", cfg, [W.TenantSpec() for _ in preds], specs))
    for i, (h, k, d, u) in enumerate(preds):
        o.sft[(i, W.GEMM)] = SFTEntry(count=1, h2d=h, kl=k, d2h=d, util=u)
        o.jobs[i].arrived = True
    for jid, gid, phase in resident:
        j = o.jobs[jid]
        o.tenants[j.tenant].pending.clear()
        o.tenants[j.tenant].inflight = 1
        j.placed, j.gid, j.phase, j.place_order = True, gid, phase, o.place_counter
        o.place_counter += 1
        o.devices[gid].resident.append(jid)
    o.admission(0)
    return [(int(f[7]), int(f[2]), int(f[9])) for f in (ln.split() for ln in o.trace) if f[1] == "PLACE"]


# ------------------------------------------------------------------ GUF (L827)
def test_guf_sums_utilisation_including_the_new_job():
    # GUF places a job where the summed GPU utilisation of the
    # device's jobs (the new one included) is lowest.  Two high-util (H, 60000
    # of 65536) and two low-util (L, 1000) jobs in the order H L H L on G=2:
    #   H0 -> GID0 (0+60000 on both, tie -> lowest GID)       score 60000
    #   L1 -> GID1 (GID0 60000+1000, GID1 0+1000)              score 1000
    #   H2 -> GID1 (GID0 60000+60000, GID1 1000+60000)         score 61000
    #   L3 -> GID0 (GID0 60000+1000, GID1 61000+1000)          score 61000
    # One of each per GPU.  (Taking a max instead of the sum would put both H
    # jobs on GID0; leaving out the new job's own term changes every score.)
    H, L = (1, 1, 1, 60000), (1, 1, 1, 1000)
    got = warm_oracle(W.GUF, 2, [H, L, H, L])
    assert got == [(0, 0, 60000), (1, 1, 1000), (2, 1, 61000), (3, 0, 61000)]


# ------------------------------------------------------------------ DTF (L829)
def test_dtf_balances_the_larger_of_copy_and_kernel_time():
    # DTF balances data-transfer time against compute time, i.e.
    # minimises max(sum copy ns, sum KL ns) on the device after adding the job.
    # Transfer-heavy T = (50, 0, 50), compute-heavy C = (0, 100, 0), order T C T C:
    #   T0 -> GID0 max(100, 0) = 100 (tie)       C1 -> GID0 max(100, 100) = 100 (tie)
    #   T2 -> GID1 max(100, 0) = 100 (GID0: 200) C3 -> GID1 max(100, 100) = 100 (GID0: 200)
    # This is the brute-force optimum of the (copy, KL) vector load: 100 on each GPU.
    # (A sum copy+KL would put T0,T2 on GID0 and C1,C3 on GID1: max load 200.)
    T, C = (50, 0, 50, 0), (0, 100, 0, 0)
    preds = [T, C, T, C]
    vec = [[h + d, k] for (h, k, d, _) in preds]
    opt, _ = bruteforce.optimal_vector_load(vec, 2)
    assert opt == 100
    for joint in (0, 1):
        got = warm_oracle(W.DTF, 2, preds, joint=joint)
        assert got == [(0, 0, 100), (1, 0, 100), (2, 1, 100), (3, 1, 100)], joint
        pl = [g for _, g, _ in sorted(got)]
        assert bruteforce.vector_load(vec, pl, 2) == opt


def test_joint_selection_ties_go_to_admission_order_then_lowest_gid():
    # R-16 / C-16: joint (job, device) selection minimises the score; equal
    # scores go to the earlier job in admission order, then the lower GID.
    # Four identical jobs (10, 10, 10) on G=2: every first choice ties.
    #   J0 -> GID0 max(20, 10) = 20;  J1 -> GID1 20 (GID0 would be 40)
    #   J2 -> GID0 max(40, 20) = 40;  J3 -> GID1 40
    got = warm_oracle(W.DTF, 2, [(10, 10, 10, 0)] * 4, joint=1)
    assert got == [(0, 0, 20), (1, 1, 20), (2, 0, 40), (3, 1, 40)]


# ------------------------------------------- remaining work of resident jobs
# Resident job 0 on GID0 has finished its H2D (phase KL): only its KL and D2H
# remain.  Resident job 1 on GID1 has not started (phase H2D).  New job 2.
RES = [(1000, 200, 300, 0), (0, 100, 500, 0), (10, 20, 30, 0)]
RES_AT = [(0, 0, KL), (1, 1, H2D)]


def test_rtf_counts_only_remaining_phases():
    # RTF uses the predicted *remaining* runtime of the jobs
    # on each GPU.  GID0: 200 + 300 (+ new 60) = 560;  GID1: 0 + 100 + 500 (+ 60) = 660.
    # (Counting job 0's finished H2D would make GID0 1560 and move the job to GID1.)
    assert warm_oracle(W.RTF, 2, RES, resident=RES_AT) == [(2, 0, 560)]


def test_dtf_counts_only_remaining_phases():
    # GID0: max(300 + 40, 200 + 20) = 340;  GID1: max(500 + 40, 100 + 20) = 540
    assert warm_oracle(W.DTF, 2, RES, resident=RES_AT) == [(2, 0, 340)]


def test_mbf_counts_only_remaining_phases():
    # PAPER.md L831 / R-13: max(sum h2d, sum d2h, sum hbm, sum sm) where a KL
    # phase splits into hbm = min(kl, ceil(180224/6000) = 31) and sm = kl - hbm.
    # Job 0 at phase D2H (only its D2H remains, say); new job 2 = (10, 20, 30):
    # hbm 20, sm 0.  GID0: max(10, 300+30, 20, 0) = 330.
    # GID1 (job 1 at phase H2D): max(0+10, 500+30, 31+20, 69+0) = 530.
    got = warm_oracle(W.MBF, 2, RES, resident=[(0, 0, D2H), (1, 1, H2D)])
    assert got == [(2, 0, 330)]


# ------------------------------------------------------------ priors (R-13)
def test_class_priors_at_nominal_rates():
    # R-13 / SURVEY §8(d): with no SFT sample a job's prediction is its class
    # prior at the fixed nominal peaks 50 B/ns (link), 6000 B/ns (HBM) and
    # 700,000 FLOP/ns (one KL slot), each rounded up; util = floor(kl*65536/total).
    #  VSCALE 2^20: 4 MiB each way -> 83,887 ns; kernel 8 MiB -> 1,399 ns;
    #               util 1399*65536 // 169173 = 541
    #  GEMM 256^3 R=64: 256 KiB each way -> 5,243 ns; 2^31 FLOP -> 3,068 ns
    #               (HBM 512 KiB -> 88 ns is smaller); util 3068*65536 // 13554 = 14834
    #  XFER 2^24:   64 MiB each way -> 1,342,178 ns; kernel 128 MiB -> 22,370 ns;
    #               util 22370*65536 // 2706726 = 541
    specs = [W.JobSpec(tenant=0, kclass=W.VSCALE, n=1 << 20),
             W.JobSpec(tenant=1, kclass=W.GEMM, m=256, n=256, k=256, reps=64),
             W.JobSpec(tenant=2, kclass=W.XFER, n=1 << 24)]
    o = Oracle(W.Workload("prior", W.SystemConfig(), [W.TenantSpec() for _ in specs], specs))
    assert o.pred(o.jobs[0]) == (83887, 1399, 83887, 541)
    assert o.pred(o.jobs[1]) == (5243, 3068, 5243, 14834)
    assert o.pred(o.jobs[2]) == (1342178, 22370, 1342178, 541)


def test_cold_resident_job_enters_rtf_score_with_its_prior():
    # A resident job with no SFT sample contributes its class prior to the
    # RTF score of a warm job (R-13).  Cold GEMM 256^3 R=64 on GID0, phase H2D:
    # 5243 + 3068 + 5243 = 13554; warm new job (1, 2, 3) -> GID1 with 6 (GID0 13560).
    cfg = W.SystemConfig(num_gpus=2, balancer=W.RTF, admit_cap=100)
    specs = [W.JobSpec(tenant=0, kclass=W.GEMM, m=256, n=256, k=256, reps=64), gemm_job(1)]
    o = Oracle(W.Workload("cold", cfg, [W.TenantSpec(), W.TenantSpec()], specs))
    o.sft[(1, W.GEMM)] = SFTEntry(count=1, h2d=1, kl=2, d2h=3, util=0)
    j0 = o.jobs[0]
    o.tenants[0].pending.clear()
    j0.placed, j0.gid, j0.phase = True, 0, H2D
    o.devices[0].resident.append(0)
    assert o.score(W.RTF, o.jobs[1], o.devices[0]) == 13560
    assert o.score(W.RTF, o.jobs[1], o.devices[1]) == 6


# --------------------------------------------------------------- SFT (R-14)
def test_sft_ewma_hand_vector():
    # R-14: one sample per completed job; the first is taken as is, then
    # v <- floor((4*sample + v)/5), the k = 0.8 of Eq. (1).
    # One tenant (c_t = 1), four jobs with phase durations (h2d, kl, d2h):
    #   (100, 1000, 10) (300, 2000, 20) (50, 500, 30) (0, 4000, 40)
    # kl  EWMA: 1000, (8000+1000)/5 = 1800, (2000+1800)/5 = 760, (16000+760)/5 = 3352
    # h2d EWMA: 100, 260, 92, 18;   d2h EWMA: 10, 18, 27, 37
    # FEEDBACK records (aux1 = h2d + d2h, aux2 = kl):
    durs = [(100, 1000, 10), (300, 2000, 20), (50, 500, 30), (0, 4000, 40)]
    jobs = [kl_only(0, k, h2d_ns=h, d2h_ns=d) for h, k, d in durs]
    o = run_oracle(W.Workload("sft", W.SystemConfig(), [W.TenantSpec()], jobs))
    fb = [(int(f[8]), int(f[9])) for f in (ln.split() for ln in o.trace) if f[1] == "FEEDBACK"]
    assert fb == [(110, 1000), (278, 1800), (119, 760), (55, 3352)]


def test_sft_util_is_kernel_share_of_the_span_from_place():
    # R-14: util = floor(KL ns * 65536 / (JOB_DONE - PLACE)).  M = 1 on one GPU:
    # job 0 (KL 1000) runs first; job 1 (KL 500) arrived at t=0 but is placed
    # only at t=1000 when job 0 leaves, and is done at 1500 -> util 65536
    # (from arrival it would be 500*65536 // 1500 = 21845).  Job 0: span 1000 -> 65536.
    # A job of its own with copies: (100, 1000, 10) -> 1000*65536 // 1110 = 59041.
    cfg = W.SystemConfig(num_gpus=1, admit_cap=1)
    o = run_oracle(W.Workload("u", cfg, [W.TenantSpec(), W.TenantSpec()], [kl_only(0, 1000), kl_only(1, 500)]))
    assert [j.t_place for j in o.jobs] == [0, 1000]
    assert o.sft[(1, W.VSCALE)].util == 65536
    o = run_oracle(W.Workload("u2", W.SystemConfig(), [W.TenantSpec()], [kl_only(0, 1000, h2d_ns=100, d2h_ns=10)]))
    assert o.sft[(0, W.VSCALE)].util == 59041


# ------------------------------------------------------------ PS fill (L819)
def ps_wakes(A, jobs):
    """jobs = [(phase, cgs)], one tenant each, all resident on GID0, nothing woken."""
    cfg = W.SystemConfig(num_gpus=1, device_policy=W.PS, partitions=3, awake_budget=A, admit_cap=64)
    o = Oracle(W.Workload("ps", cfg, [W.TenantSpec() for _ in jobs], [kl_only(i, 100) for i in range(len(jobs))]))
    d = o.devices[0]
    for i, (ph, cgs) in enumerate(jobs):
        j = o.jobs[i]
        o.tenants[i].cgs = cgs
        o.tenants[i].pending.clear()
        j.arrived = j.placed = True
        j.gid, j.phase, j.place_order = 0, ph, i
        d.resident.append(i)
    o.dispatch(0, d)
    return [(int(f[7]), f[3]) for f in (ln.split() for ln in o.trace) if f[1] == "WAKE"]


def test_ps_fill_merges_copy_candidates_by_key():
    # PAPER.md L819 / R-11: after the diversity step (one op per phase, copies in
    # min-key order), the remaining budget takes KL candidates, then H2D and D2H
    # candidates *merged* by key (H2D = D2H in the paper's priority list).
    # No KL; H2D keys 5, 8; D2H keys 1, 6; A = 3:
    #   diversity: D2H(key 1) then H2D(key 5); fill: D2H(key 6) before H2D(key 8)
    got = ps_wakes(3, [(H2D, 5), (H2D, 8), (D2H, 1), (D2H, 6)])
    assert got == [(2, "D2H"), (0, "H2D"), (3, "D2H")]


def test_ps_fill_takes_kl_before_copies():
    # KL > H2D = D2H in the fill step: KL keys 7, 9; H2D keys 1, 2; A = 4:
    #   diversity: KL(7), H2D(1); fill: KL(9), then H2D(2)
    got = ps_wakes(4, [(KL, 7), (KL, 9), (H2D, 1), (H2D, 2)])
    assert got == [(0, "KL"), (2, "H2D"), (1, "KL"), (3, "H2D")]


# ------------------------------------------------------------- Eq. (1) (L695)
def test_eq1_counts_service_still_in_progress_at_the_boundary():
    # R-6 / C-6: GS of an epoch includes the part of a running op inside it.
    # One KL op of 12 ms on Q = 1 ms: every epoch 1..12 sees GS = 1 ms although
    # the op completes only at 12 ms.  CGS_n = floor((4*(GS<<16) + CGS_{n-1})/5):
    #   GS<<16 = 65,536,000,000;  n=1: 4*65,536,000,000/5 = 52,428,800,000
    #   n=2: (262,144,000,000 + 52,428,800,000)/5 = 62,914,560,000
    #   n=3: (262,144,000,000 + 62,914,560,000)/5 = 65,011,712,000
    cfg = W.SystemConfig(num_gpus=1, device_policy=W.FIFO, quantum_ns=1_000_000)
    o = run_oracle(W.Workload("ep", cfg, [W.TenantSpec()], [kl_only(0, 12_000_000)]))
    ep = [(int(f[0]), int(f[8]), int(f[9])) for f in (ln.split() for ln in o.trace) if f[1] == "EPOCH"]
    assert len(ep) == 12
    assert [t for t, _, _ in ep] == [n * 1_000_000 for n in range(1, 13)]
    assert all(gs == 1_000_000 for _, gs, _ in ep)
    assert [c for _, _, c in ep[:3]] == [52_428_800_000, 62_914_560_000, 65_011_712_000]


def test_eq1_partial_epoch_service_splits_at_the_boundary():
    # An op from 0.4 ms to 1.6 ms (H2D 0.4 ms of another tenant first) with Q = 1 ms:
    # tenant 1's GS = 0.6 ms in epoch 1 and 0.6 ms in epoch 2.
    #   CGS_1 = 4*(600000<<16)/5 = 31,457,280,000
    #   CGS_2 = (157,286,400,000 + 31,457,280,000)/5 = 37,748,736,000
    cfg = W.SystemConfig(num_gpus=1, device_policy=W.FIFO, partitions=1, awake_budget=1, quantum_ns=1_000_000)
    # (a third tenant's job arriving at 2.5 ms keeps the clock running past 2 ms)
    jobs = [kl_only(0, 400_000), kl_only(1, 1_200_000), kl_only(2, 1, arrival=2_500_000)]
    o = run_oracle(W.Workload("ep2", cfg, [W.TenantSpec()] * 3, jobs))
    ep = [(int(f[0]), int(f[8]), int(f[9])) for f in (ln.split() for ln in o.trace)
          if f[1] == "EPOCH" and f[5] == "1"]
    assert ep[:2] == [(1_000_000, 600_000, 31_457_280_000), (2_000_000, 600_000, 37_748_736_000)]


# ------------------------------------------------- LAS at the balancer (L693)
def _las_admission_blocks(weights):
    """Two tenants, 30 identical 100 us KL-only jobs each, all at t = 0, one
    resident job at a time (M = 1), weighted-LAS admission, Q = 1 ms.  Returns
    the tenant of each PLACE in order."""
    cfg = W.SystemConfig(num_gpus=1, partitions=1, awake_budget=1, admit_cap=1, balancer=W.GMIN,
                         las_admission=1, device_policy=W.FIFO, quantum_ns=1_000_000)
    jobs = [kl_only(t, 100_000) for _ in range(30) for t in (0, 1)]
    o = run_oracle(W.Workload("las", cfg, [W.TenantSpec(weight=w) for w in weights], jobs))
    return [int(f[5]) for f in (ln.split() for ln in o.trace) if f[1] == "PLACE"]


def test_las_admission_alternates_whole_epochs_between_equal_tenants():
    # PAPER.md L693-695 + R-7: the LAS key is the decayed service CGS, which only
    # changes at epoch boundaries; within an epoch the lower key keeps winning.
    # Epoch 1: both CGS = 0, tie -> tenant 0 takes all 10 admissions (1 ms / 100 us).
    # At 1 ms: CGS_0 = 4*(1e6 << 16)/5 = 52,428,800,000 > CGS_1 = 0 -> tenant 1's epoch;
    # at 2 ms: CGS_0 = 52,428,800,000/5 = 10,485,760,000 < CGS_1 = 52,428,800,000 -> tenant 0 ...
    seq = _las_admission_blocks((1, 1))
    assert seq[:40] == [0] * 10 + [1] * 10 + [0] * 10 + [1] * 10


def test_las_admission_weights_divide_the_decayed_service():
    # R-7: a before b iff CGS_a * p_b < CGS_b * p_a.  Weights 8 : 1, per epoch:
    #   1: tie 0 = 0 -> tenant 0         CGS = (52,428,800,000, 0)
    #   2: 52.4e9 * 1 > 0 * 8 -> 1       CGS = (10,485,760,000, 52,428,800,000)
    #   3: 10.5e9 * 1 < 52.4e9 * 8 -> 0  CGS = (54,525,952,000, 10,485,760,000)
    #   4: 54.5e9 * 1 < 10.5e9 * 8 -> 0  CGS = (63,333,990,400, 2,097,152,000)
    #   5: 63.3e9 * 1 > 2.1e9 * 8 -> 1
    # (with k = 0.8 the decay is steep, so a weight of 8 buys 2 epochs of 3, not 8 of 9)
    seq = _las_admission_blocks((8, 1))
    assert seq[:50] == [0] * 10 + [1] * 10 + [0] * 20 + [1] * 10


def test_c4c_admissions_are_capacity_blocked():
    # the contention variant exists to exercise LAS at the balancer: jobs that
    # had arrived wait for a device with room (c_t = 4 x 64 tenants vs M = 4 x 8)
    wl = W.config_c4c()
    o = Oracle(wl)
    blocked = []
    orig = o.admission

    def counted(t):
        orig(t)
        # the admission loop stopped; if an eligible job is left, no device had room
        elig = [tn for tn in o.tenants if tn.pending and tn.inflight < tn.c and o.jobs[tn.pending[0]].arrived]
        if elig:
            blocked.append(t)
    o.admission = counted
    o.run()
    assert len(blocked) > 100
    base = Oracle(W.config_c4())                 # the BASELINE C4 never blocks on capacity
    orig_b, blocked_b = base.admission, []

    def counted_b(t):
        orig_b(t)
        if any(tn.pending and tn.inflight < tn.c and base.jobs[tn.pending[0]].arrived for tn in base.tenants):
            blocked_b.append(t)
    base.admission = counted_b
    base.run()
    assert blocked_b == []


# ------------------------------------------------------- arbiter (L311, L1073; R-15)
def _placements(o):
    """(job, gid, tenant, policy, score) of every PLACE record, in order."""
    return [(int(f[7]), int(f[2]), int(f[5]), int(f[8]), int(f[9]))
            for f in (ln.split() for ln in o.trace) if f[1] == "PLACE"]


def test_arbiter_places_cold_jobs_by_gmin():
    # PAPER.md L311, L1073 (reading R-15): a feedback policy needs a sample of the
    # job's (tenant, class) in the SFT; until then the arbiter places it by GMin.
    # G = 2, RTF, three cold jobs at t = 0: a 64 MiB XFER (tenant 0), then two
    # tiny VSCALE jobs (tenants 1, 2).  GMin: XFER -> GID0 (0 / 0 resident, tie),
    # VSCALE -> GID1 (1 / 0), VSCALE -> GID0 (1 / 1, tie -> lowest GID); the
    # scores are the resident counts 0, 0, 1 and every PLACE records GMIN (1).
    # (RTF on the class priors would send the third job to GID1, away from the
    # XFER's ~2.7 ms of predicted remaining transfer time.)
    cfg = W.SystemConfig(num_gpus=2, balancer=W.RTF, admit_cap=10 ** 6)
    specs = [W.JobSpec(tenant=0, kclass=W.XFER, n=1 << 24),
             W.JobSpec(tenant=1, kclass=W.VSCALE, n=1024),
             W.JobSpec(tenant=2, kclass=W.VSCALE, n=1024)]
    o = Oracle(W.Workload("pin", cfg, [W.TenantSpec() for _ in specs], specs))
    for j in o.jobs:
        j.arrived = True
    o.admission(0)
    assert _placements(o) == [(0, 0, 0, W.GMIN, 0), (1, 1, 1, W.GMIN, 0), (2, 0, 2, W.GMIN, 1)]


def test_dynamic_is_mbf_once_the_class_has_a_sample():
    # R-15: DYNAMIC places a (tenant, class) with MBF once the SFT holds a sample
    # of it, and a class without one by GMin.  G = 2, no joint selection; tenant
    # 0's GEMM row is warm, tenant 1's cold: PLACE records MBF (6) for tenant 0's
    # job and GMIN (1) for tenant 1's.
    cfg = W.SystemConfig(num_gpus=2, balancer=W.DYNAMIC, admit_cap=10 ** 6, joint_select=0)
    specs = [gemm_job(0), gemm_job(1)]
    o = Oracle(W.Workload("pin", cfg, [W.TenantSpec() for _ in specs], specs))
    o.sft[(0, W.GEMM)] = SFTEntry(count=1, h2d=10, kl=20, d2h=10, util=30000)
    for j in o.jobs:
        j.arrived = True
    o.admission(0)
    assert {t: pol for (_, _, t, pol, _) in _placements(o)} == {0: W.MBF, 1: W.GMIN}


# ------------------------------------------ FIFO dispatch and arrival-order admission
def _records(trace, kind):
    lines = trace.splitlines() if isinstance(trace, str) else trace
    return [ln.split() for ln in lines if ln.split()[1] == kind]


def test_fifo_wakes_in_placement_order():
    # The FIFO device policy (the CUDA-runtime-like baseline) wakes ready
    # phases in the order their jobs were PLACED, not by tenant id.  One GPU, awake
    # budget A = 1.  Job A (tenant 1) arrives at 0, job B (tenant 0) at 10; every
    # phase 100 / 50 / 100 ns.  A's H2D holds the one wake until t = 100; then A's
    # KL and B's H2D are both ready and A, placed first, goes first:
    #   t=0 A H2D, 100 A KL, 150 A D2H, 250 B H2D, 350 B KL, 400 B D2H.
    # (Waking by tenant would start B's H2D at t = 100.)
    cfg = W.SystemConfig(num_gpus=1, balancer=W.GMIN, device_policy=W.FIFO, awake_budget=1, admit_cap=4)
    jobs = [kl_only(1, 50, arrival=0, h2d_ns=100, d2h_ns=100), kl_only(0, 50, arrival=10, h2d_ns=100, d2h_ns=100)]
    wl = W.Workload("pin", cfg, [W.TenantSpec(), W.TenantSpec()], jobs)
    got = [(int(f[0]), int(f[5]), f[3]) for f in _records(run_oracle(wl).trace, "WAKE")]
    assert got == [(0, 1, "H2D"), (100, 1, "KL"), (150, 1, "D2H"), (250, 0, "H2D"), (350, 0, "KL"), (400, 0, "D2H")]


def test_arrival_order_admission_is_by_arrival_then_tenant():
    # Admission without LAS takes pending jobs in arrival order (DESIGN
    # §4.4: (arrival, tenant, seq)).  One GPU with room for one job (M = 1): job C
    # (tenant 2) arrives at 0 and holds the slot until its H2D ends at 100 (KL and
    # D2H take 0); job D (tenant 1) arrives at 10, job E (tenant 0) at 20.  At 100
    # D, the earlier arrival, is placed, then E at 200:
    #   PLACE t=0 tenant 2, t=100 tenant 1, t=200 tenant 0.
    # (Ordering by tenant first would place E before D.)
    cfg = W.SystemConfig(num_gpus=1, balancer=W.GMIN, device_policy=W.PS, admit_cap=1)
    jobs = [kl_only(2, 0, arrival=0, h2d_ns=100), kl_only(1, 0, arrival=10, h2d_ns=100),
            kl_only(0, 0, arrival=20, h2d_ns=100)]
    wl = W.Workload("pin", cfg, [W.TenantSpec() for _ in range(3)], jobs)
    got = [(int(f[0]), int(f[5])) for f in _records(run_oracle(wl).trace, "PLACE")]
    assert got == [(0, 2), (100, 1), (200, 0)]
