"""Figs 14/15 analogue on the pairwise mix (NEXT-2), in virtual time.

For each pair A..I (strings_workload.PAIRS) and each balancer, the scheduler's
schedule is computed with injected (nominal) phase durations -- by the oracle
DES, which the C++ core reproduces byte for byte (so this is exactly what the
library decides; on a GPU in INJECTED timing it executes the same schedule).
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
from oracle.des import run_oracle  # noqa: E402

POLICIES = [W.GRR, W.GMIN, W.GWTMIN, W.RTF, W.GUF, W.DTF, W.MBF, W.DYNAMIC]


def mean_lat(o):
    acc = {}
    for j in o.jobs:
        acc.setdefault(j.tenant, []).append(j.t_jobdone - j.arrival)
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
                o = run_oracle(W.config_pair(idx, seed=seed, num_gpus=args.gpus, balancer=p))
                lat = mean_lat(o)
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
