"""Per-job phase timeline of C1's VSCALE chains in MEASURED timing (host clock, us):
where a chain step's time goes (H2D, KL, D2H, the gap to the next job's H2D)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import strings_workload as W
from paper_conf_sc_senguptagsp14_b200 import strings as S
from paper_conf_sc_senguptagsp14_b200.runner import run_workload
wl = W.config_c1()
for rep in range(3):
    r = run_workload(wl, timing_mode=S.MEASURED)
rows = []
for spec, inf in zip(wl.jobs, r.infos):
    rows.append((spec.tenant, inf.seq, inf.gid, inf.t_place, list(inf.t_start), list(inf.t_done),
                 inf.kl_gpu_start_ns, inf.kl_gpu_end_ns))
t0 = min(x[3] for x in rows)
print("eager jobs", r.stats.eager_jobs, "span us", (max(x[5][2] for x in rows) - t0) / 1e3)
for t in range(4):
    prev = None
    for ten, seq, gid, tp, st, dn, k0, k1 in sorted(x for x in rows if x[0] == t):
        f = lambda v: round((v - t0) / 1e3, 1)
        gap = None if prev is None else round((st[0] - prev) / 1e3, 1)
        print(json.dumps({"t": ten, "s": seq, "g": gid, "place": f(tp), "h2d": [f(st[0]), f(dn[0])],
                          "kl": [f(st[1]), f(dn[1])], "d2h": [f(st[2]), f(dn[2])], "gap_prev_d2h_to_h2d": gap,
                          "kl_dev_us": round((k1 - k0) / 1e3, 1) if k1 else None}))
        prev = dn[2]
