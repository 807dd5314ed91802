"""The plain C oracle kernels (oracle/c/kernels.c, bench's cpu_baseline) agree
with the numpy oracle (oracle/kernels.py), which tests/test_oracle_kernels.py
pins to published vectors and closed forms -- no GPU."""
import numpy as np
import pytest

import strings_workload as W
from oracle import cbind
from oracle import kernels as K


@pytest.mark.parametrize("n", [0, 1, 5, 4099, 1 << 16])
def test_vscale_xfer_scan_hist_bit_exact(n):
    rng = np.random.default_rng(n)
    x = rng.uniform(-1, 1, n).astype(np.float32)
    x[::7] = np.float32(1e-41)                            # denormals pass through the multiply
    assert np.array_equal(cbind.vscale(x, 1.0009765625).view(np.uint32), K.vscale(x, 1.0009765625).view(np.uint32))
    u = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    assert np.array_equal(cbind.xfer(u, 0x9E3779B9), K.xfer(u, 0x9E3779B9))
    assert np.array_equal(cbind.scan(u), K.scan(u))
    b = rng.integers(0, 256, n).astype(np.uint8)
    assert np.array_equal(cbind.hist(b), K.hist(b))


def test_sort_segments_exact():
    x = np.random.default_rng(3).integers(0, 1 << 32, 2048 * 5, dtype=np.uint64).astype(np.uint32)
    assert np.array_equal(cbind.sort_segments(x), K.sort_segments(x))


@pytest.mark.parametrize("int_valued", [True, False])
def test_gemm_matches_the_double_accumulated_oracle(int_valued):
    spec = W.JobSpec(tenant=0, kclass=W.GEMM, m=64, n=48, k=80, data_seed=11, int_valued=int_valued)
    a, b = W.job_inputs(spec)
    ref = K.gemm(a, b)
    got = cbind.gemm(a, b, reps=3)
    if int_valued:
        assert np.array_equal(got, ref)                   # every partial sum is an exact integer
    else:
        # both sum exact products in double and round once; only the summation
        # order differs (numpy's BLAS), so they agree to within one float ulp
        assert np.all(np.abs(got.astype(np.float64) - ref) <= np.spacing(np.abs(ref).astype(np.float32)))


def test_job_runner_runs_every_job_in_tenant_order():
    wl = W.config_c1(reps=2, scale=64)
    ins = [W.job_inputs(s) for s in wl.jobs]
    outs = [[np.zeros(sh, dt) for sh, dt in W.job_output_shapes(s)] for s in wl.jobs]
    cbind.run_jobs(wl.jobs, ins, outs, threads=3)
    for s, i, o in zip(wl.jobs, ins, outs):
        want = K.run_job(s, i)[0]
        if s.kclass == W.GEMM:
            assert np.all(np.abs(o[0].astype(np.float64) - want) <= np.spacing(np.abs(want).astype(np.float32)))
        else:
            assert np.array_equal(o[0].view(np.uint32), want.view(np.uint32))
