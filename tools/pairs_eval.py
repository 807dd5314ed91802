"""Figs 14/15 analogue on the pairwise mix (NEXT-2), in virtual time.

For each pair A..I (strings_workload.PAIRS) and each balancer, the schedule is
computed with injected (nominal) phase durations by the library's own decision
core in DECISIONS_ONLY mode (no device needed; on a GPU in INJECTED timing the
library executes exactly this schedule, and tests/ pin it to the oracle).
Weighted speedup of a policy = mean over tenants of (mean latency under GRR /
mean latency under the policy) (reading R-1, baseline = GRR as in the paper's
Figs 12-15).  Prints one JSON line per pair and a summary.

    python tools/pairs_eval.py [--gpus 2] [--seeds 3]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import strings_workload as W  # noqa: E402
from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402
from paper_conf_sc_senguptagsp14_b200.runner import run_workload  # noqa: E402

POLICIES = [W.GRR, W.GMIN, W.GWTMIN, W.RTF, W.GUF, W.DTF, W.MBF, W.DYNAMIC]


def mean_lat(res):
    acc = {}
    for i in res.infos:
        acc.setdefault(i.tenant, []).append(i.t_done[2] - i.t_arrival)
    return {t: statistics.mean(v) for t, v in acc.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=2)
    ap.add_argument("--seeds", type=int, default=3)
    args = ap.parse_args()
    summary = {W.BALANCER_NAMES[p]: [] for p in POLICIES}
    for idx, (a, b) in enumerate(W.PAIRS):
        row = {"pair": f"{chr(65 + idx)}:{a}-{b}"}
        ws_by_pol = {p: [] for p in POLICIES}
        for seed in range(1, args.seeds + 1):
            base = None
            for p in POLICIES:
                r = run_workload(W.config_pair(idx, seed=seed, num_gpus=args.gpus, balancer=p),
                                 timing_mode=S.DECISIONS_ONLY)
                lat = mean_lat(r)
                if p == W.GRR:
                    base = lat
                ws_by_pol[p].append(sum(base[t] / lat[t] for t in lat) / len(lat))
        for p in POLICIES:
            v = statistics.mean(ws_by_pol[p])
            row[W.BALANCER_NAMES[p]] = round(v, 3)
            summary[W.BALANCER_NAMES[p]].append(v)
        print(json.dumps(row), flush=True)
    print(json.dumps({"mean_weighted_speedup_vs_GRR": {k: round(statistics.mean(v), 3) for k, v in summary.items()},
                      "gpus": args.gpus, "seeds": args.seeds, "timing": "virtual (injected nominal durations)"}))


if __name__ == "__main__":
    main()
