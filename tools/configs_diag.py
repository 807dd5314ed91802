"""Where does the time go in a measured multi-logical-device config?

Runs one BASELINE config (node mode: G logical devices on the visible GPUs,
MEASURED timing, caller-pinned buffers) through the library and reports, from
the per-job records (strings_job_info):
  * span, effective host-link GB/s per direction;
  * union occupancy of the physical copy engines: the fraction of the span in
    which >= 1 H2D (resp. D2H) op of ANY logical device was running;
  * per class: p50 phase durations and the GB/s a single op achieved;
  * mean concurrency of H2D ops (how many logical devices copy at once).

    python tools/configs_diag.py C4 [--awake-budget A] [--policy LAS|PS|...]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import strings_workload as W  # noqa: E402
from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402


def union_len(iv):
    iv = sorted(iv)
    tot, cur_s, cur_e = 0, None, None
    for s, e in iv:
        if cur_e is None or s > cur_e:
            if cur_e is not None:
                tot += cur_e - cur_s
            cur_s, cur_e = s, e
        else:
            cur_e = max(cur_e, e)
    if cur_e is not None:
        tot += cur_e - cur_s
    return tot


def main():
    import torch
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--awake-budget", type=int, default=0)
    ap.add_argument("--policy", default=None)
    ap.add_argument("--gpus", type=int, default=0, help="logical devices (0 = the config's)")
    ap.add_argument("--repeats", type=int, default=2)
    ap.add_argument("--trace", default=None, help="write the last repeat's decision trace here")
    args = ap.parse_args()
    wl = W.CONFIGS[args.config]()
    cfg = wl.config
    if args.gpus:
        cfg.num_gpus = args.gpus
    if args.awake_budget:
        cfg.awake_budget = args.awake_budget
        cfg.admit_cap = 2 * args.awake_budget
    if args.policy:
        cfg.device_policy = W.DEVICE_POLICY_NAMES.index(args.policy)
    cfg = cfg.resolved()
    ngpu = torch.cuda.device_count()
    need_in, need_out = {}, {}
    for sp in wl.jobs:
        need_in[sp.tenant] = [max(a, b) for a, b in zip(need_in.get(sp.tenant, [0, 0]), (sp.h2d_sizes() + [0])[:2])]
        need_out[sp.tenant] = max(need_out.get(sp.tenant, 0), sum(sp.d2h_sizes()))
    hin = {t: [torch.empty(max(1, b), dtype=torch.uint8).pin_memory() for b in v] for t, v in need_in.items()}
    hout = {t: torch.empty(max(1, b), dtype=torch.uint8).pin_memory() for t, b in need_out.items()}
    for rep in range(args.repeats):
        S.init_from_config(cfg, timing_mode=S.MEASURED, physical_gpus=ngpu, trace_in_memory=False,
                           trace_path=args.trace if rep == args.repeats - 1 else None)
        ts = [S.register_tenant(t.weight, t.max_inflight) for t in wl.tenants]
        t0 = time.perf_counter()
        for sp in wl.jobs:
            ins = [S.HostRef(hin[sp.tenant][i].data_ptr(), b) for i, b in enumerate(sp.h2d_sizes())]
            outs = [S.HostRef(hout[sp.tenant].data_ptr(), b) for b in sp.d2h_sizes()]
            S.submit_spec(ts[sp.tenant], sp, ins, outs)
        st = S.drain()
        wall = time.perf_counter() - t0
        infos = [S.job_info(i) for i in range(len(wl.jobs))]
        stats = S.stats()
        S.shutdown()
    t_first = min(i.t_arrival for i in infos)
    t_last = max(i.t_done[2] for i in infos)
    span = t_last - t_first
    h2d_b = sum(sum(sp.h2d_sizes()) for sp in wl.jobs)
    d2h_b = sum(sum(sp.d2h_sizes()) for sp in wl.jobs)
    res = {"config": args.config, "logical_gpus": cfg.num_gpus, "physical_gpus": ngpu,
           "device_policy": W.DEVICE_POLICY_NAMES[cfg.device_policy], "A": cfg.awake_budget, "M": cfg.admit_cap,
           "status": st, "span_ms": round(span / 1e6, 2), "wall_ms": round(wall * 1e3, 2),
           "jobs_per_s": round(len(infos) / (span / 1e9), 1),
           "h2d_GBps": round(h2d_b / span, 2), "d2h_GBps": round(d2h_b / span, 2),
           "decision_us_per_job": round((stats.decision_ns - stats.issue_ns) / 1e3 / len(infos), 2),
           "issue_us_per_job": round(stats.issue_ns / 1e3 / len(infos), 2)}
    for x, name in ((0, "h2d"), (1, "kl"), (2, "d2h")):
        iv = [(i.t_start[x], i.t_done[x]) for i in infos if i.t_done[x] > i.t_start[x]]
        res[f"{name}_union_occupancy"] = round(union_len(iv) / span, 4)
        res[f"{name}_mean_concurrency"] = round(sum(e - s for s, e in iv) / max(1, union_len(iv)), 2)
    # KL path under load: host issue -> leader claim -> body start -> last CTA -> host observe
    off = stats.gpu_clock_offset_ns[0]
    for cname in sorted({W.CLASS_NAMES[sp.kclass] for sp in wl.jobs}):
        ii = [i for sp, i in zip(wl.jobs, infos) if W.CLASS_NAMES[sp.kclass] == cname and i.kl_gpu_start_ns]
        if not ii or not off:
            continue

        def med(v):
            v = sorted(v)
            return round(v[len(v) // 2] / 1e3, 1)
        res[f"{cname}_kl_path_us_p50"] = {
            "issue_to_claim": med([i.kl_gpu_start_ns - off - i.kl_host_issue_ns for i in ii]),
            "claim_to_exec": med([i.kl_gpu_exec_ns - i.kl_gpu_start_ns for i in ii]),
            "exec_to_end": med([i.kl_gpu_end_ns - i.kl_gpu_exec_ns for i in ii]),
            "end_to_observe": med([i.kl_host_observe_ns - (i.kl_gpu_end_ns - off) for i in ii]),
            "model_start_to_done": med([i.t_done[1] - i.t_start[1] for i in ii])}
    by = {}
    for sp, i in zip(wl.jobs, infos):
        d = by.setdefault(W.CLASS_NAMES[sp.kclass], {"h2d": [], "kl": [], "d2h": [], "wait": [], "bytes": sum(sp.h2d_sizes())})
        d["h2d"].append(i.t_done[0] - i.t_start[0])
        d["kl"].append(i.t_done[1] - i.t_start[1])
        d["d2h"].append(i.t_done[2] - i.t_start[2])
        d["wait"].append(i.t_start[0] - i.t_arrival)
    for c, d in by.items():
        p50 = {k: sorted(v)[len(v) // 2] / 1e3 for k, v in d.items() if k != "bytes"}
        res[c] = {f"{k}_us_p50": round(v, 1) for k, v in p50.items()}
        res[c]["h2d_op_GBps_p50"] = round(d["bytes"] / (p50["h2d"] * 1e3), 2) if p50["h2d"] else None
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
