"""C-ABI library on a host without a GPU: symbols, loud failure, host-logic parity.

The decision core (C++, libstrings_sched.so) is host logic; DECISIONS_ONLY mode
replays it without any device work so its traces can be compared with the
independent CPU oracle here.  Product timing modes must fail loudly (ECUDA)
when no CUDA device exists.
"""
import ctypes
import os
import subprocess

import numpy as np
import pytest

import strings_workload as W
from oracle import invariants
from oracle.des import run_oracle
from paper_conf_sc_senguptagsp14_b200 import strings as S
from paper_conf_sc_senguptagsp14_b200.runner import run_workload


def _has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def test_library_exports_every_declared_symbol():
    declared = S.declared_symbols()
    assert len(declared) >= 17
    out = subprocess.run(["nm", "-D", "--defined-only", S.LIB_PATH], capture_output=True, text=True,
                         check=True).stdout
    exported = {ln.split()[-1] for ln in out.splitlines() if " T " in ln}
    missing = [s for s in declared if s not in exported]
    assert missing == []
    for s in declared:
        assert hasattr(S.lib, s)


def test_version_and_strerror():
    assert "sm_100a" in S.version()
    assert S.strerror(S.EINVAL) == "invalid argument"
    assert S.strerror(S.EFAULT).startswith("a job")


@pytest.mark.skipif(_has_gpu(), reason="checks the no-GPU failure path")
def test_product_modes_fail_loudly_without_gpu():
    for mode in (S.MEASURED, S.INJECTED):
        with pytest.raises(S.StringsError) as e:
            S.init(timing_mode=mode)
        assert e.value.status == S.ECUDA


def test_calls_before_init_are_rejected():
    assert S.lib.strings_sync(0) == S.ESTATE
    assert S.lib.strings_drain() == S.ESTATE
    assert S.lib.strings_shutdown() == S.ESTATE


def test_argument_validation():
    S.init(num_gpus=1, timing_mode=S.DECISIONS_ONLY)
    try:
        t = S.register_tenant(1, 1)
        x = np.zeros(16, np.float32)
        y = np.zeros(16, np.float32)
        with pytest.raises(S.StringsError):                      # wrong byte count
            S.submit(t, S.make_desc(S.VSCALE, n=8), [x], [y])
        with pytest.raises(S.StringsError):                      # unknown tenant
            S.submit(t + 5, S.make_desc(S.VSCALE, n=16), [x], [y])
        a = np.zeros((128, 64), np.uint16)
        b = np.zeros((64, 200), np.uint16)
        c = np.zeros((128, 200), np.float32)
        with pytest.raises(S.StringsError):                      # n % 256 != 0
            S.submit(t, S.make_desc(S.GEMM, m=128, n=200, k=64), [a, b], [c])
        with pytest.raises(S.StringsError):                      # missing buffer
            S.submit(t, S.make_desc(S.GEMM, m=128, n=256, k=64), [a], [c])
        with pytest.raises(S.StringsError):
            S.submit(t, S.make_desc(7, n=16), [x], [y])
        assert S.sync(t) == S.OK
        with pytest.raises(S.StringsError):
            S.register_tenant(0, 1)
    finally:
        S.shutdown()
    with pytest.raises(S.StringsError):
        S.init(balancer=11, timing_mode=S.DECISIONS_ONLY)


@pytest.mark.parametrize("name", list(W.CONFIGS))
def test_decision_core_trace_matches_oracle_on_configs(name):
    wl = W.CONFIGS[name]()
    o = run_oracle(wl)
    r = run_workload(wl, timing_mode=S.DECISIONS_ONLY)
    assert r.status == S.OK
    assert r.trace == o.trace
    assert r.stats.jobs_done == len(wl.jobs)


@pytest.mark.parametrize("seed", range(150))
def test_decision_core_trace_matches_oracle_on_random_workloads(seed):
    wl = W.random_workload(seed)
    o = run_oracle(wl)
    r = run_workload(wl, timing_mode=S.DECISIONS_ONLY)
    assert r.trace == o.trace


def test_decision_core_job_records_match_oracle():
    wl = W.config_c4(jobs_per_tenant=4)
    o = run_oracle(wl)
    r = run_workload(wl, timing_mode=S.DECISIONS_ONLY)
    for j, info in zip(o.jobs, r.infos):
        assert info.gid == j.gid
        assert list(info.t_start) == j.start and list(info.t_done) == j.done
        assert info.status == S.OK
    assert invariants.check(r.trace, wl) == []


def test_trace_file_written(tmp_path):
    wl = W.config_c1()
    p = tmp_path / "trace.txt"
    r = run_workload(wl, timing_mode=S.DECISIONS_ONLY, trace_path=str(p))
    assert p.read_text().splitlines() == r.trace


def test_sync_per_tenant_and_unregister():
    S.init(num_gpus=2, timing_mode=S.DECISIONS_ONLY)
    try:
        ts = [S.register_tenant(1, 1) for _ in range(3)]
        dummy = np.zeros(16, np.uint8)
        for t in ts:
            for s in range(4):
                d = S.make_desc(S.VSCALE, n=1 << 20, arrival_ns=0, inj=(1000 * (t + 1), 500, 1000))
                S.submit(t, d, [S.HostRef(dummy.ctypes.data, 4 << 20)], [S.HostRef(dummy.ctypes.data, 4 << 20)])
        assert S.sync(ts[0]) == S.OK
        assert S.unregister_tenant(ts[1]) == S.OK
        with pytest.raises(S.StringsError):
            S.submit(ts[1], S.make_desc(S.VSCALE, n=4), [np.zeros(4, np.float32)], [np.zeros(4, np.float32)])
        assert S.drain() == S.OK
        st = S.stats()
        assert st.jobs_done == 12 and st.jobs_failed == 0
    finally:
        S.shutdown()


@pytest.mark.parametrize("weights,slice_ns", [((1, 1), 500_000), ((2, 1), 200_000), ((1, 3), 1)])
def test_tfs_fair_share_trace_matches_oracle(weights, slice_ns):
    cfg = W.SystemConfig(num_gpus=1, partitions=1, device_policy=W.TFS, admit_cap=1000, tfs_slice_ns=slice_ns)
    jobs = []
    for t, size in ((0, 200_000), (1, 50_000)):
        jobs += [W.JobSpec(tenant=t, kclass=W.VSCALE, n=0, inj_kl_ns=size) for _ in range(60)]
    wl = W.Workload("tfs", cfg, [W.TenantSpec(weight=w, max_inflight=1000) for w in weights], jobs)
    o = run_oracle(wl)
    r = run_workload(wl, timing_mode=S.DECISIONS_ONLY)
    assert r.trace == o.trace
    assert invariants.check(r.trace, wl) == []


@pytest.mark.parametrize("name", ["C1", "C3", "C5"])
def test_tfs_on_configs_matches_oracle(name):
    wl = W.CONFIGS[name]()
    wl.config.device_policy = W.TFS
    assert run_workload(wl, timing_mode=S.DECISIONS_ONLY).trace == run_oracle(wl).trace


def test_slot_size_and_mode_validation():
    S.init(num_gpus=1, timing_mode=S.DECISIONS_ONLY, slot_bytes=1 << 20)
    try:
        t = S.register_tenant()
        big = S.HostRef(1, 4 << 20)
        with pytest.raises(S.StringsError) as e:      # 4 MiB in + 4 MiB out > 1 MiB slot
            S.submit(t, S.make_desc(S.VSCALE, n=1 << 20), [big], [big])
        assert e.value.status == S.EINVAL
    finally:
        S.shutdown()
    for bad in (dict(kl_mode=2), dict(device_policy=4), dict(balancer=-1)):
        with pytest.raises(S.StringsError):
            S.init(timing_mode=S.DECISIONS_ONLY, **bad)
    with pytest.raises(S.StringsError) as e:
        S.init(timing_mode=3)
    assert e.value.status == S.EINVAL
    # device-side limits: A <= kRing (256) KL ring entries, M <= 0xFFFF (16-bit slot of a lent share)
    for bad in (dict(awake_budget=257), dict(admit_cap=65536)):
        with pytest.raises(S.StringsError) as e:
            S.init(timing_mode=S.DECISIONS_ONLY, **bad)
        assert e.value.status == S.EINVAL
    S.init(timing_mode=S.DECISIONS_ONLY, awake_budget=256, admit_cap=512)
    S.shutdown()


def test_heterogeneous_gwtmin_parity_and_validation():
    wl = W.config_c3()
    wl.config.balancer = W.GWTMIN
    wl.config.device_weights = [3, 2, 2, 1]
    o = run_oracle(wl)
    r = run_workload(wl, timing_mode=S.DECISIONS_ONLY)
    assert r.trace == o.trace
    # the first placements at t=0 follow load/weight: the weight-3 device gets 3 of the first 8
    first8 = [int(l.split()[2]) for l in r.trace if " PLACE " in l][:8]
    assert first8.count(0) == 3 and first8.count(3) == 1
    with pytest.raises(S.StringsError) as e:
        S.init(num_gpus=2, timing_mode=S.DECISIONS_ONLY, device_weights=[1, 0])
    assert e.value.status == S.EINVAL


@pytest.mark.parametrize("pair", range(9))
def test_pairwise_mix_trace_matches_oracle(pair):
    for bal in (W.GMIN, W.DTF, W.MBF):
        wl = W.config_pair(pair, balancer=bal)
        assert run_workload(wl, timing_mode=S.DECISIONS_ONLY).trace == run_oracle(wl).trace


def test_product_path_never_imports_the_oracle():
    # oracle/ is test infrastructure: the package, tools and the bench's main leg
    # must not import it (bench.py may only in its cpu_baseline / reference legs)
    import ast
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    files = [os.path.join(d, f) for sub in ("paper_conf_sc_senguptagsp14_b200", "tools", "strings_workload")
             for d, _, fs in os.walk(os.path.join(root, sub)) for f in fs if f.endswith(".py")]
    for path in files:
        tree = ast.parse(open(path).read())
        for node in ast.walk(tree):
            if isinstance(node, (ast.Import, ast.ImportFrom)):
                names = [a.name for a in node.names] + ([node.module] if isinstance(node, ast.ImportFrom) else [])
                assert not any(n and n.split(".")[0] == "oracle" for n in names), path
    allowed = {"cpu_baseline", "_oracle_shard", "run_reference"}
    tree = ast.parse(open(os.path.join(root, "bench.py")).read())
    for fn in [n for n in tree.body if isinstance(n, ast.FunctionDef)]:
        for node in ast.walk(fn):
            if isinstance(node, ast.ImportFrom) and node.module and node.module.split(".")[0] == "oracle":
                assert fn.name in allowed, fn.name


@pytest.mark.parametrize("pyname,cname", [("Config", "strings_config_t"), ("KernelDesc", "strings_kernel_desc_t"),
                                          ("Buf", "strings_buf_t"), ("JobInfo", "strings_job_info_t"),
                                          ("Stats", "strings_stats_t")])
def test_binding_structs_match_the_header_layout(pyname, cname, tmp_path):
    # the ctypes mirrors in strings.py must have the C structs' size and every
    # field at the C offset (a drifted binding would read or write past the struct)
    st = getattr(S, pyname)
    names = [f[0] for f in st._fields_]
    src = tmp_path / "layout.c"
    body = "\n".join(f'  printf("%zu\\n", offsetof({cname}, {n}));' for n in names)
    src.write_text(f'#include <stdio.h>\n#include <stddef.h>\n#include "strings_sched.h"\n'
                   f'int main(void) {{\n  printf("%zu\\n", sizeof({cname}));\n{body}\n  return 0;\n}}\n')
    exe = tmp_path / "layout"
    inc = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include")
    subprocess.run(["gcc", "-std=c11", "-I", inc, str(src), "-o", str(exe)], check=True)
    out = [int(v) for v in subprocess.run([str(exe)], check=True, capture_output=True, text=True).stdout.split()]
    assert out[0] == ctypes.sizeof(st), (cname, out[0], ctypes.sizeof(st))
    assert out[1:] == [getattr(st, n).offset for n in names], cname


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4c", "C5"])
def test_library_defaults_match_the_readings(name):
    # A = 2 + P (R-11), M = 2A (R-12), joint selection on for DTF/MBF/DYNAMIC (R-16):
    # the library's own defaulting (strings_init with 0 / -1) gives the oracle's trace
    wl = W.CONFIGS[name]()
    assert wl.config.awake_budget == 0 and wl.config.joint_select == -1
    r = run_workload(wl, timing_mode=S.DECISIONS_ONLY, library_defaults=True)
    assert r.trace == run_oracle(wl).trace
