"""Figs 14/15 analogue on the pairwise mix (NEXT-2), MEASURED on the B200.

Like tools/pairs_eval.py, but every pair runs on the GPU in MEASURED timing: a
submitter thread calls strings_submit at each job's Eq. (4) arrival time
(P:L885-889), dilated by the number of logical devices per GPU so the offered
load per physical host link is the pair's; latency = JOB_DONE - submit.  For
each pair A..I and balancer: weighted speedup over GRR (reading R-1: mean over
tenants of GRR's mean latency / the policy's; the paper's Figs 12-15 baseline).

    python tools/pairs_measured.py [--gpus 2] [--seeds 2]
"""
import argparse
import dataclasses
import json
import os
import statistics
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import strings_workload as W  # noqa: E402
from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402

POLICIES = [W.GRR, W.GMIN, W.GWTMIN, W.RTF, W.GUF, W.DTF, W.MBF, W.DYNAMIC]


def run_pair(wl, ngpu, bufs):
    cfg = wl.config.resolved()
    S.init_from_config(cfg, timing_mode=S.MEASURED, physical_gpus=ngpu, trace_in_memory=False)
    ts = [S.register_tenant(t.weight, t.max_inflight) for t in wl.tenants]
    ids = [None] * len(wl.jobs)

    def submitter():
        t0 = time.perf_counter_ns()
        for i, sp in enumerate(wl.jobs):
            due = t0 + sp.arrival_ns
            while time.perf_counter_ns() < due:
                pass
            ins, outs = bufs[(sp.tenant, sp.kclass)]
            ids[i] = S.submit_spec(ts[sp.tenant], sp, ins, outs)
    th = threading.Thread(target=submitter)
    th.start()
    th.join()
    st = S.drain()
    infos = [S.job_info(j) for j in ids]
    S.shutdown()
    assert st == S.OK, st
    lat = {}
    for i in infos:
        lat.setdefault(i.tenant, []).append((i.t_done[2] - i.t_arrival) / 1e6)
    return {t: statistics.mean(v) for t, v in lat.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=2)
    ap.add_argument("--seeds", type=int, default=2)
    args = ap.parse_args()
    ngpu = torch.cuda.device_count()
    dil = max(1, -(-args.gpus // ngpu))
    summary = {W.BALANCER_NAMES[p]: [] for p in POLICIES}
    for idx, (a, b) in enumerate(W.PAIRS):
        row = {"pair": f"{chr(65 + idx)}:{a}-{b}"}
        ws = {p: [] for p in POLICIES}
        for seed in range(1, args.seeds + 1):
            base = None
            for p in POLICIES:
                wl = W.config_pair(idx, seed=seed, num_gpus=args.gpus, balancer=p)
                wl = dataclasses.replace(wl, jobs=[dataclasses.replace(j, arrival_ns=j.arrival_ns * dil)
                                                   for j in wl.jobs])
                bufs = {}
                for sp in wl.jobs:
                    key = (sp.tenant, sp.kclass)
                    if key not in bufs:
                        bufs[key] = ([torch.from_numpy(x.view(np.uint8).reshape(-1)).pin_memory()
                                      for x in W.job_inputs(sp)],
                                     [torch.empty(n, dtype=torch.uint8).pin_memory() for n in sp.d2h_sizes()])
                lat = run_pair(wl, ngpu, bufs)
                if p == W.GRR:
                    base = lat
                ws[p].append(sum(base[t] / lat[t] for t in lat) / len(lat))
        for p in POLICIES:
            v = statistics.mean(ws[p])
            row[W.BALANCER_NAMES[p]] = round(v, 3)
            summary[W.BALANCER_NAMES[p]].append(v)
        print(json.dumps(row), flush=True)
    print(json.dumps({"mean_weighted_speedup_vs_GRR": {k: round(statistics.mean(v), 3) for k, v in summary.items()},
                      "logical_gpus": args.gpus, "physical_gpus": ngpu, "seeds": args.seeds,
                      "timing": "MEASURED, open loop (Eq. (4) arrivals dilated x%d)" % dil}), flush=True)


if __name__ == "__main__":
    main()
