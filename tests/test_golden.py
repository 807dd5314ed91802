"""Golden fixtures (tests/golden/, each file cites its source) checked against the oracle."""
import os

import numpy as np
import pytest

import strings_workload as W
from oracle import kernels as K
from oracle.des import D2H, H2D, KL, Oracle, run_oracle

GOLD = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
PHASE = {"H2D": H2D, "KL": KL, "D2H": D2H}
POL = {"PS": W.PS, "LAS": W.LAS, "FIFO": W.FIFO}


def rows(name):
    for ln in open(os.path.join(GOLD, name)):
        ln = ln.split("#")[0].strip()
        if ln:
            yield ln


def _ps_state(policy, A, cands):
    cfg = W.SystemConfig(num_gpus=1, device_policy=policy, partitions=3, awake_budget=A, admit_cap=64)
    specs = [W.JobSpec(tenant=i, kclass=W.VSCALE, n=0, inj_kl_ns=100) for i in range(len(cands))]
    o = Oracle(W.Workload("g", cfg, [W.TenantSpec() for _ in cands], specs))
    d = o.devices[0]
    for i, (ph, cgs) in enumerate(cands):
        j = o.jobs[i]
        o.tenants[i].cgs = cgs
        o.tenants[i].pending.clear()
        j.arrived = j.placed = True
        j.gid, j.phase, j.place_order = 0, ph, i
        d.resident.append(i)
    o.dispatch(0, d)
    return sorted(f"{int(f[7])}:{f[3]}" for f in (l.split() for l in o.trace) if f[1] == "WAKE")


@pytest.mark.parametrize("line", list(rows("ps_worked_cases.txt")))
def test_ps_worked_cases(line):
    lhs, rhs = line.split("->")
    f = lhs.split()
    cands = [(PHASE[c.split(":")[0]], int(c.split(":")[1])) for c in f[2:]]
    assert _ps_state(POL[f[0]], int(f[1]), cands) == sorted(rhs.split())


def test_eq1_worked_decay():
    cfg = W.SystemConfig(num_gpus=1, device_policy=W.FIFO, partitions=2, quantum_ns=10_000_000)
    jobs = [W.JobSpec(tenant=0, kclass=W.VSCALE, n=0, inj_kl_ns=10_000_000),
            W.JobSpec(tenant=1, kclass=W.VSCALE, n=0, inj_kl_ns=1, arrival_ns=35_000_000)]
    o = run_oracle(W.Workload("eq1", cfg, [W.TenantSpec(), W.TenantSpec()], jobs))
    ep = {int(f[0]) // 1_000_000: (int(f[8]), int(f[9])) for f in (l.split() for l in o.trace)
          if f[1] == "EPOCH" and f[5] == "0"}
    for line in rows("eq1_decay.txt"):
        t, gs, cgs = line.split()
        g, c = ep[int(t)]
        assert g == int(gs) * 1_000_000
        assert abs(c / 65536 - float(cgs) * 1e6) <= 1.0


def test_hash_and_prng_vectors():
    for line in rows("hash_prng_vectors.txt"):
        f = line.split()
        if f[0] == "fmix32":
            assert int(K.fmix32(np.array([int(f[1], 16)], np.uint32))[0]) == int(f[2], 16)
        else:
            r = W.SplitMix64(int(f[1]))
            assert [r.next_u64() for _ in f[2:]] == [int(x) for x in f[2:]]


def test_paper_headline_arithmetic():
    # the headline speedups are the per-figure ratios times GRR-Rain's 2.16x (L891)
    for line in rows("paper_relative_numbers.txt"):
        _, ratio, headline = line.split()
        assert abs(float(ratio) * 2.16 - float(headline)) < 0.02
