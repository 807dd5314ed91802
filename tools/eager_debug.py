"""Run C1 in MEASURED timing with a short stall dump (debugging eager chaining)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("STRINGS_STALL_DUMP_S", "3")
import strings_workload as W
from paper_conf_sc_senguptagsp14_b200 import strings as S
from paper_conf_sc_senguptagsp14_b200.runner import run_workload
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 2
wl = W.config_c1(reps=reps)
if len(sys.argv) > 2 and sys.argv[2] == "vscale_only":
    wl.jobs = [j for j in wl.jobs if j.kclass == W.VSCALE]
r = run_workload(wl, timing_mode=S.MEASURED)
print("status", r.status, "eager jobs", r.stats.eager_jobs)
