"""Full-size BASELINE configs C1, C3, C4 and C5 through the C ABI on the B200.

The configs at the sizes BASELINE.json names (2,048 and 3,072 jobs, 64 MiB XFER
buffers) do not fit the per-job buffers tests/test_gpu_scheduler.py gives
every job, so here the inputs of each (tenant, class) are generated once and
reused by all jobs of that class of tenants t, t + 8, ..., non-sampled jobs write into
one scratch output per class, and a sample of jobs (spread over classes,
tenants, devices and time) gets outputs of its own that are checked against
the oracle's CPU kernels on the same input bytes.

* INJECTED timing: the decision trace is byte-identical to the oracle's DES of
  the full workload; every op still runs on the GPU.
* MEASURED timing (the mode bench.py times): the trace satisfies the
  invariants I1-I5/I7.
Outputs: VSCALE and XFER bit-exact (XFER on 64 Ki sampled elements plus both
ends of the buffer), GEMM within 1e-5 normwise (C-22).
"""
import numpy as np
import pytest

import strings_workload as W
from oracle import invariants
from oracle import kernels as K
from gemm_bounds import gemm_elementwise_ok
from oracle.des import run_oracle
from paper_conf_sc_senguptagsp14_b200 import strings as S

pytestmark = pytest.mark.gpu


def _sample(wl, k):
    """About k jobs: the first and last of every class plus an even spread."""
    pick = set()
    by_cls = {}
    for i, j in enumerate(wl.jobs):
        by_cls.setdefault(j.kclass, []).append(i)
    for ids in by_cls.values():
        pick.update((ids[0], ids[-1]))
        step = max(1, len(ids) // max(1, k // len(by_cls)))
        pick.update(ids[::step])
    return sorted(pick)


def _run(wl, timing, sample):
    import torch
    cfg = wl.config.resolved()
    nphys = torch.cuda.device_count()
    arenas = S.torch_arenas(cfg.num_gpus, min(nphys, cfg.num_gpus), cfg.admit_cap, 0)
    S.init_from_config(cfg, timing_mode=timing, physical_gpus=len(arenas), arenas=arenas,
                       trace_in_memory=True)
    pinned = []

    def pin(a):
        p = S.pinned_array(a.shape, a.dtype)
        p[...] = a
        pinned.append(p)
        return p

    try:
        for t in wl.tenants:
            S.register_tenant(t.weight, t.max_inflight)
        shared_in, scratch_out = {}, {}
        ins_of, outs_of = [], []
        for i, spec in enumerate(wl.jobs):
            key = (spec.tenant % 8, spec.kclass)      # inputs shared by tenants t, t+8, ...: bounded pinned memory
            if key not in shared_in:
                shared_in[key] = [pin(a) for a in W.job_inputs(spec)]
            if spec.kclass not in scratch_out:
                scratch_out[spec.kclass] = [pin(np.zeros(s, d)) for s, d in W.job_output_shapes(spec)]
            ins_of.append(shared_in[key])
            outs_of.append([pin(np.zeros(s, d)) for s, d in W.job_output_shapes(spec)]
                           if i in sample else scratch_out[spec.kclass])
        for i, spec in enumerate(wl.jobs):
            S.submit_spec(spec.tenant, spec, ins_of[i], outs_of[i])
        status = S.drain()
        trace = S.trace()
        infos = [S.job_info(i) for i in range(len(wl.jobs))]
        got = {i: [np.array(o, copy=True) for o in outs_of[i]] for i in sample}
        used = {i: [np.array(a, copy=True) for a in ins_of[i]] for i in sample}
    finally:
        S.shutdown()
        for a in pinned:
            S.free_pinned(a)
        del arenas
    return status, trace, infos, got, used


def _check_outputs(wl, got, used):
    rng = np.random.default_rng(1)
    for i, outs in got.items():
        spec, ins = wl.jobs[i], used[i]
        if spec.kclass == W.XFER:                 # the whole 2^24-element output
            assert np.array_equal(outs[0], K.xfer(ins[0], spec.seed)), i
            continue
        want = K.run_job(spec, ins)
        for g, r in zip(outs, want):
            if spec.kclass == W.GEMM and not spec.int_valued:
                err = np.max(np.abs(g.astype(np.float64) - r)) / np.max(np.abs(r))
                assert err <= 1e-5, (i, err)
                assert gemm_elementwise_ok(g, ins[0], ins[1]), i
            else:
                assert np.array_equal(g.view(np.uint32), r.view(np.uint32)), i


@pytest.mark.parametrize("name", ["C1", "C3", "C4", "C5", "C4c"])
@pytest.mark.parametrize("timing", [S.INJECTED, S.MEASURED])
def test_full_size_config(name, timing):
    wl = W.CONFIGS[name]()
    sample = set(_sample(wl, 24))
    status, trace, infos, got, used = _run(wl, timing, sample)
    assert status == S.OK
    assert all(inf.status == S.OK for inf in infos)
    if timing == S.INJECTED:
        assert trace == run_oracle(wl).trace
    else:
        assert invariants.check(trace, wl) == []
    # every job was placed, and its KL ran on a partition of the persistent kernel
    assert all(0 <= inf.gid < wl.config.num_gpus and inf.kl_partition >= 0 for inf in infos)
    _check_outputs(wl, got, used)
