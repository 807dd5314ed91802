"""Mutation check of the oracle's pins -- no GPU.

Each entry below is a plausible slip in ``oracle/`` (a sum where the paper's
rule needs a max, a dropped term, a wrong EWMA weight, a tie broken the wrong
way, ...).  The test copies the oracle, the input generator and the oracle's
pin tests into a scratch directory, applies ONE slip, and runs the pins there:
at least one pin must fail.  A slip that survives means the oracle's arithmetic
at that spot is checked only against itself -- exactly what the pins exist to
prevent (the GPU path is compared with the oracle, so a misreading shared by
both would otherwise go unseen).

The snippets are matched literally and must occur exactly once, so a refactor
of the oracle breaks this test loudly instead of silently skipping a mutation.
"""
import os
import shutil
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name, file, original snippet, mutated snippet)
MUTATIONS = [
    ("guf_sum_to_max", "oracle/des.py",
     "return sum(self.pred(i)[3] for i in res) + self.pred(j)[3]",
     "return max([self.pred(i)[3] for i in res] + [self.pred(j)[3]])"),
    ("guf_drops_new_job", "oracle/des.py",
     "return sum(self.pred(i)[3] for i in res) + self.pred(j)[3]",
     "return sum(self.pred(i)[3] for i in res)"),
    ("prior_flop_rate", "oracle/des.py",
     "PRIOR_KL_FLOP_PER_NS = 700_000", "PRIOR_KL_FLOP_PER_NS = 70_000"),
    ("prior_util_copy_share", "oracle/des.py",
     "return h, k, d, (k * 65536 // tot) if tot else 0",
     "return h, k, d, ((h + d) * 65536 // tot) if tot else 0"),
    ("sft_ewma_weight", "oracle/des.py",
     "e.kl = (4 * smp[1] + e.kl) // 5", "e.kl = (smp[1] + 4 * e.kl) // 5"),
    ("ps_fill_not_merged", "oracle/des.py",
     "for j in self.las_sorted(by[H2D] + by[D2H]):", "for j in by[H2D] + by[D2H]:"),
    ("ps_diversity_tie_to_d2h", "oracle/des.py",
     "if len(copies) == 2 and self.las_key_less(by[D2H][0], by[H2D][0]):",
     "if len(copies) == 2 and not self.las_key_less(by[H2D][0], by[D2H][0]):"),
    ("dtf_max_to_sum", "oracle/des.py",
     "return max(copy + h + dd, kern + k)", "return copy + h + dd + kern + k"),
    ("rtf_total_not_remaining", "oracle/des.py",
     "s += (h if i.phase <= H2D else 0) + (k if i.phase <= KL else 0) + (dd if i.phase <= D2H else 0)",
     "s += h + k + dd"),
    ("mbf_total_not_remaining", "oracle/des.py",
     "if fresh or i.phase <= H2D:", "if True:"),
    ("epoch_drops_in_progress", "oracle/des.py",
     "inprog[j.tenant] += t - max(j.start[x], self.epoch_start)", "inprog[j.tenant] += 0"),
    ("eq1_k_0_6", "oracle/des.py",
     "tn.cgs = (4 * (gs << 16) + old) // 5", "tn.cgs = (3 * (gs << 16) + 2 * old) // 5"),
    ("joint_tie_last", "oracle/des.py",
     "if best is None or s_ < best[0]:", "if best is None or s_ <= best[0]:"),
    ("score_tie_highest_gid", "oracle/des.py",
     "if bs is None or s < bs:", "if bs is None or s <= bs:"),
    ("util_span_from_arrival", "oracle/des.py",
     "span = t - j.t_place", "span = t - j.arrival"),
    ("tfs_no_service_history", "oracle/des.py",
     "d.svc[j.tenant] = d.svc.get(j.tenant, 0) + (t - j.start[x])", "d.svc[j.tenant] = 0"),
    ("las_admission_to_arrival", "oracle/des.py",
     "if self.cfg.las_admission:", "if False:"),
    ("las_weight_ignored", "oracle/des.py",
     "lhs, rhs = ca * b.prio, cb * a.prio", "lhs, rhs = ca, cb"),
    ("arbiter_cold_uses_feedback", "oracle/des.py",
     "if b in (W.RTF, W.GUF, W.DTF, W.MBF, W.DYNAMIC) and not self.has_sample(j):",
     "if b in (W.RTF, W.GUF, W.DTF, W.MBF, W.DYNAMIC) and False:"),
    ("dynamic_means_dtf", "oracle/des.py",
     "        if b == W.DYNAMIC:\n            return W.MBF", "        if b == W.DYNAMIC:\n            return W.DTF"),
    ("grr_cursor_not_advanced", "oracle/des.py",
     "self.grr_cursor = (g + 1) % self.G", "self.grr_cursor = g"),
    ("ct_off_by_one", "oracle/des.py",
     "if tn.pending and tn.inflight < tn.c:", "if tn.pending and tn.inflight <= tn.c:"),
    ("admit_cap_off_by_one", "oracle/des.py",
     "adm = [d for d in self.devices if len(d.resident) < self.M]",
     "adm = [d for d in self.devices if len(d.resident) <= self.M]"),
    ("awake_budget_off_by_one", "oracle/des.py",
     "free = self.A - d.woken_unfinished", "free = self.A - d.woken_unfinished + 1"),
    ("fifo_wakes_by_tenant", "oracle/des.py",
     "for j in sorted(cands, key=lambda j: j.place_order)[:free]:",
     "for j in sorted(cands, key=lambda j: (j.tenant, j.seq))[:free]:"),
    ("las_wake_most_service_first", "oracle/des.py",
     "for j in self.las_sorted(cands)[:free]:", "for j in self.las_sorted(cands)[::-1][:free]:"),
    ("ps_no_kl_diversity", "oracle/des.py",
     "if active[KL] == 0 and by[KL] and free > 0:", "if False:"),
    ("las_tie_highest_tenant", "oracle/des.py",
     "return -1 if a.tenant < b.tenant else 1", "return -1 if a.tenant > b.tenant else 1"),
    ("arrival_order_by_tenant_first", "oracle/des.py",
     "return sorted(js, key=lambda j: (j.arrival, j.tenant, j.seq))",
     "return sorted(js, key=lambda j: (j.tenant, j.arrival, j.seq))"),
    ("tfs_slice_ignores_weight", "oracle/des.py",
     "if d.awake is None or d.awake_used >= self.tenants[d.awake].weight * self.S:",
     "if d.awake is None or d.awake_used >= self.S:"),
    ("tfs_pick_most_service", "oracle/des.py",
     "if best is None or d.svc.get(tid, 0) * self.tenants[best].weight < \\",
     "if best is None or d.svc.get(tid, 0) * self.tenants[best].weight > \\"),
    ("sft_first_sample_averaged_with_zero", "oracle/des.py",
     "        if e.count == 0:\n            e.h2d, e.kl, e.d2h, e.util = smp[0], smp[1], smp[2], util",
     "        if e.count == 0:\n            e.h2d, e.kl, e.d2h, e.util = (4 * smp[0]) // 5, (4 * smp[1]) // 5, (4 * smp[2]) // 5, (4 * util) // 5"),
    ("one_kl_slot", "oracle/des.py",
     "self.busy = [[None], [None] * self.P, [None]]", "self.busy = [[None], [None], [None]]"),
    ("epoch_service_from_start_not_epoch", "oracle/des.py",
     "tn.gs_acc += t - max(j.start[x], self.epoch_start)", "tn.gs_acc += t - j.start[x]"),
    ("gwtmin_ignores_weight", "oracle/des.py",
     "if best is None or len(d.resident) * best.weight < len(best.resident) * d.weight:",
     "if best is None or len(d.resident) < len(best.resident):"),
    ("fmix32_shift", "oracle/kernels.py",
     "h ^= h >> np.uint32(13)", "h ^= h >> np.uint32(15)"),
    ("gemm_rounds_operands_to_f32", "oracle/kernels.py",
     "return (a @ b).astype(np.float32)",
     "return (a.astype(np.float32) @ b.astype(np.float32)).astype(np.float32)"),
    ("jain_unsquared_sum", "oracle/metrics.py",
     "return sum(xs) ** 2 / (n * s2)", "return sum(xs) / (n * s2)"),
    ("ws_inverted", "oracle/metrics.py",
     "return sum(b / p for b, p in zip(base_lat, policy_lat)) / len(base_lat)",
     "return sum(p / b for b, p in zip(base_lat, policy_lat)) / len(base_lat)"),
    ("tstar_no_chain", "oracle/metrics.py",
     "terms.append(max(v / inflight.get(t, 1) for t, v in chains.items()))", "pass"),
    ("tstar_hbm_only", "oracle/metrics.py",
     'sum(j["hbm"] + j["h2d"] + j["d2h"] for j in jobs) / bm,', 'sum(j["hbm"] for j in jobs) / bm,'),
    ("tstar_no_arrival", "oracle/metrics.py",
     'terms.append(max(j.get("arrival", 0.0) + j["h2d"] / bh + klstar(j) + j["d2h"] / bd for j in jobs) - t0)',
     "pass"),
    ("bruteforce_max", "oracle/bruteforce.py", "if best is None or v < best:", "if best is None or v > best:"),
    ("inv_no_I4_admission", "oracle/invariants.py",
     'errs.append(f"I4 tenant {tn} placed job {j} before {pending[tn][0]}")', "pass"),
    ("inv_M_off_by_one", "oracle/invariants.py", "if len(resident[g]) > M:", "if len(resident[g]) > M + 1:"),
    ("inv_no_I5_budget", "oracle/invariants.py",
     'errs.append(f"I5 t={t} gid={g} {len(c)} candidates unwoken with budget {A - woken_unf[g]}")', "pass"),
    ("inv_no_I5_idle", "oracle/invariants.py",
     'errs.append(f"I5 t={t} gid={g} engine {x} idle with woken op")', "pass"),
    ("inv_no_I4_start", "oracle/invariants.py",
     'errs.append(f"I4 tenant {ten_of[j]} engine {x} job {j} started after a later job")', "pass"),
    ("inv_no_I7", "oracle/invariants.py",
     'errs.append(f"I7 t={r.t} gid={g} TFS woke tenant {ten_of[j]} while {others} awake")', "pass"),
]

PIN_FILES = ["test_oracle_pins.py", "test_oracle_des.py", "test_golden.py",
             "test_oracle_metrics.py", "test_oracle_kernels.py"]


def _stage(dst):
    for d in ("oracle", "strings_workload"):
        shutil.copytree(os.path.join(ROOT, d), os.path.join(dst, d),
                        ignore=shutil.ignore_patterns("__pycache__"))
    os.makedirs(os.path.join(dst, "tests"))
    for f in ["conftest.py", "gemm_bounds.py"] + PIN_FILES:
        shutil.copy(os.path.join(ROOT, "tests", f), os.path.join(dst, "tests", f))
    shutil.copytree(os.path.join(ROOT, "tests", "golden"), os.path.join(dst, "tests", "golden"))
    shutil.copy(os.path.join(ROOT, "pytest.ini"), os.path.join(dst, "pytest.ini"))


def _run_pins(dst):
    env = dict(os.environ, PYTHONPATH=dst, PYTHONDONTWRITEBYTECODE="1")
    cmd = [sys.executable, "-m", "pytest", "-x", "-q", "-m", "not slow and not gpu",
           "-p", "no:cacheprovider"] + [os.path.join("tests", f) for f in PIN_FILES]
    return subprocess.run(cmd, cwd=dst, env=env, capture_output=True, text=True, timeout=900)


def test_every_mutation_is_caught_by_a_pin(tmp_path):
    base = tmp_path / "base"
    _stage(str(base))
    # the unmutated copy must pass every pin file (so a failure below is the
    # mutation's, never the harness's)
    r = _run_pins(str(base))
    assert r.returncode == 0, r.stdout[-2000:]

    def one(m):
        name, path, old, new = m
        dst = tmp_path / name
        _stage(str(dst))
        fp = dst / path
        src = fp.read_text()
        assert src.count(old) == 1, f"{name}: snippet not found exactly once in {path}"
        fp.write_text(src.replace(old, new))
        r = _run_pins(str(dst))
        return name, r.returncode, r.stdout[-1500:]

    muts = MUTATIONS
    assert len(muts) >= 30
    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 2)) as ex:
        results = list(ex.map(one, muts))
    survivors = [(n, rc, out) for n, rc, out in results if rc != 1]
    # rc 1 = some test failed; 0 = the mutation survived; anything else = harness error
    assert not survivors, "\n".join(f"{n}: rc={rc}\n{out}" for n, rc, out in survivors)
