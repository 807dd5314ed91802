"""Tenant kernel parity on the B200 (stand-alone launches through the C ABI).

Each kernel is launched through ``strings_kernel_launch`` (the same device
bodies the persistent dispatcher runs) on torch-allocated device memory and
compared element by element with the CPU oracle (oracle/kernels.py):
VSCALE and XFER bit-exact, GEMM bit-exact on integer-valued inputs and within
1e-5 normwise relative error on random inputs (reading R-22).
"""
import numpy as np
import pytest

import strings_workload as W
from oracle import kernels as K
from gemm_bounds import gemm_elementwise_ok
from paper_conf_sc_senguptagsp14_b200 import strings as S

pytestmark = pytest.mark.gpu


def _torch():
    import torch
    return torch


def _launch(desc, ins, outs, ctas=0):
    torch = _torch()
    dev_in = [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in ins]
    dev_out = [torch.zeros(o.nbytes, dtype=torch.uint8, device="cuda") for o in outs]
    S.kernel_launch(0, desc, [t.data_ptr() for t in dev_in], [t.data_ptr() for t in dev_out], ctas=ctas,
                    stream=torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    return [t.cpu().numpy().view(o.dtype).reshape(o.shape) for t, o in zip(dev_out, outs)]


@pytest.mark.parametrize("n", [0, 1, 3, 4, 5, 1023, 4097, 65536 + 7, (1 << 20) + 3, 1 << 24])
@pytest.mark.parametrize("ctas", [0, 1, 37])
def test_vscale_bit_exact(n, ctas):
    rng = np.random.default_rng(n + 17)
    x = rng.uniform(-1, 1, n).astype(np.float32)
    if n > 8:
        x[:4] = np.array([1e-45, -2.0 ** -126, 3.4e38, -0.0], dtype=np.float32)   # denormal, huge, -0
    a = 1.0 + 2.0 ** -10
    (y,) = _launch(S.make_desc(S.VSCALE, n=n, alpha=a), [x], [np.zeros(n, np.float32)], ctas)
    assert np.array_equal(y.view(np.uint32), K.vscale(x, a).view(np.uint32))


@pytest.mark.parametrize("n", [0, 1, 7, 4096, 65537, (1 << 22) + 1])
def test_xfer_bit_exact(n):
    rng = np.random.default_rng(n + 3)
    x = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    seed = 0xDEADBEEF
    (y,) = _launch(S.make_desc(S.XFER, n=n, seed=seed), [x], [np.zeros(n, np.uint32)])
    assert np.array_equal(y, K.xfer(x, seed))


def test_streaming_unaligned_pointers():
    torch = _torch()
    n = 10_001
    x = np.random.default_rng(1).uniform(-1, 1, n + 1).astype(np.float32)
    dx = torch.from_numpy(x).cuda()
    dy = torch.zeros(n + 1, dtype=torch.float32, device="cuda")
    S.kernel_launch(0, S.make_desc(S.VSCALE, n=n, alpha=3.0), [dx.data_ptr() + 4], [dy.data_ptr() + 4],
                    stream=torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert np.array_equal(dy.cpu().numpy()[1:].view(np.uint32), K.vscale(x[1:], 3.0).view(np.uint32))


def _gemm_inputs(m, n, k, seed, int_valued):
    rng = np.random.default_rng(seed)
    if int_valued:
        a = rng.integers(-2, 3, (m, k)).astype(np.float32)
        b = rng.integers(-2, 3, (k, n)).astype(np.float32)
    else:
        a = rng.uniform(-1, 1, (m, k)).astype(np.float32)
        b = rng.uniform(-1, 1, (k, n)).astype(np.float32)
    return W.f32_to_bf16_bits(a), W.f32_to_bf16_bits(b)


@pytest.mark.parametrize("m,n,k", [(128, 256, 64), (256, 256, 256), (384, 512, 128), (128, 768, 192)])
@pytest.mark.parametrize("reps,ctas", [(1, 0), (3, 2), (64, 5), (7, 148)])
def test_gemm_integer_inputs_bit_exact(m, n, k, reps, ctas):
    a, b = _gemm_inputs(m, n, k, m * 7 + n + k, True)
    (c,) = _launch(S.make_desc(S.GEMM, m=m, n=n, k=k, reps=reps), [a, b], [np.zeros((m, n), np.float32)], ctas)
    assert np.array_equal(c, K.gemm(a, b))


@pytest.mark.parametrize("m,n,k", [(128, 256, 64), (256, 256, 256), (512, 256, 256)])
def test_gemm_random_inputs_within_tolerance(m, n, k):
    a, b = _gemm_inputs(m, n, k, 99 + m, False)
    (c,) = _launch(S.make_desc(S.GEMM, m=m, n=n, k=k, reps=2), [a, b], [np.zeros((m, n), np.float32)])
    ref = K.gemm(a, b)
    err = np.max(np.abs(c.astype(np.float64) - ref)) / np.max(np.abs(ref))
    assert err <= 1e-5, err
    assert gemm_elementwise_ok(c, a, b)


def test_gemm_structured_operands_catch_layout_errors():
    # A = I-like selector, B = arange: C rows must pick exact B rows (catches
    # transposed / mis-strided smem layouts that random data might average out)
    m, n, k = 128, 256, 128
    a = np.zeros((m, k), np.float32)
    for i in range(m):
        a[i, (i * 5) % k] = 1.0
    b = (np.arange(k * n) % 251 - 125).astype(np.float32).reshape(k, n)
    ab, bb = W.f32_to_bf16_bits(a), W.f32_to_bf16_bits(b)
    (c,) = _launch(S.make_desc(S.GEMM, m=m, n=n, k=k, reps=1), [ab, bb], [np.zeros((m, n), np.float32)])
    assert np.array_equal(c, K.gemm(ab, bb))


# ------------------------------------------------ NEXT-2: HIST / SCAN / SORT
@pytest.mark.parametrize("n", [0, 1, 15, 16, 4097, 1_000_003, 1 << 24])
@pytest.mark.parametrize("ctas", [0, 1, 37])
def test_hist_bit_exact(n, ctas):
    spec = W.JobSpec(tenant=0, kclass=W.HIST, n=n, data_seed=n + ctas)
    (x,) = W.job_inputs(spec)
    (h,) = _launch(S.make_desc(S.HIST, n=n), [x], [np.zeros(256, np.uint32)], ctas)
    assert np.array_equal(h, K.hist(x))


def test_hist_single_bin_contention():
    x = np.full(1 << 20, 7, np.uint8)
    (h,) = _launch(S.make_desc(S.HIST, n=x.size), [x], [np.zeros(256, np.uint32)])
    assert h[7] == x.size and h.sum() == x.size


@pytest.mark.parametrize("ctas", [1, 3])
def test_hist_one_bin_large_share(ctas):
    # one CTA counts > 2^24 copies of one byte (per-lane counters far past 16 bits)
    # through the bulk pipeline, plus a ragged tail on the LDG / byte paths
    n = (1 << 24) * 2 // ctas + 77
    x = np.full(n, 200, np.uint8)
    x[::4097] = 3
    (h,) = _launch(S.make_desc(S.HIST, n=n), [x], [np.zeros(256, np.uint32)], ctas)
    assert np.array_equal(h, K.hist(x))


@pytest.mark.parametrize("ctas", [2, 37])
@pytest.mark.parametrize("offset", [0, 3])
def test_hist_bulk_path(ctas, offset):
    # 41 whole 32 KB chunks per CTA through the TMA bulk pipeline (chunks dealt
    # round-robin over the CTAs, 4 stages cycling several times); 4099 tail bytes
    # go through the 16-B and byte loads.  offset 3: the same bytes from an
    # unaligned start (byte loads only)
    torch = _torch()
    n = ctas * 41 * 32768 + 4099
    spec = W.JobSpec(tenant=0, kclass=W.HIST, n=n + offset, data_seed=ctas + offset)
    (x,) = W.job_inputs(spec)
    dx = torch.from_numpy(x).cuda()
    out = torch.zeros(256, dtype=torch.int32, device="cuda")
    S.kernel_launch(0, S.make_desc(S.HIST, n=n), [dx.data_ptr() + offset], [out.data_ptr()], ctas=ctas,
                    stream=torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().view(np.uint32), K.hist(x[offset:]))


@pytest.mark.parametrize("n", [0, 1, 7, 8, 2047, 2049, 100_003, (1 << 22) + 5])
@pytest.mark.parametrize("ctas", [0, 1, 5, 148])
def test_scan_bit_exact(n, ctas):
    x = np.random.default_rng(n).integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    (y,) = _launch(S.make_desc(S.SCAN, n=n), [x], [np.zeros(n, np.uint32)], ctas)
    assert np.array_equal(y, K.scan(x))


# The aligned SCAN body works in waves of about STRINGS_SCAN_WAVE_MB (16 MB) split
# over the CTAs, with a wave's sums published two waves ahead: these sizes give
# 3-5 waves (so the interleaved sum(k+2) path and the 8-row tag ring both run),
# ragged last sub-blocks and CTAs with nothing in the last wave.
@pytest.mark.parametrize("n,ctas", [(3 * (1 << 22) + 5, 1), ((1 << 24) + 9, 5), ((1 << 25) + 3, 37),
                                    ((1 << 25) - 4, 148), (5 * (1 << 22), 1)])
def test_scan_bit_exact_multi_wave(n, ctas):
    x = np.random.default_rng(n).integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    (y,) = _launch(S.make_desc(S.SCAN, n=n), [x], [np.zeros(n, np.uint32)], ctas)
    assert np.array_equal(y, K.scan(x))


def test_scan_back_to_back_items_reuse_the_wave_table():
    # consecutive launches on the same group state: each item's wave words carry
    # a fresh tag, so a small item never reads a big item's stale words
    torch = _torch()
    st = torch.cuda.current_stream()
    sizes = [(1 << 24) + 3, 100, 1 << 22, 8193, (1 << 24) + 3, 0, 5 * (1 << 22) + 1]
    xs, ys = [], []
    for i, n in enumerate(sizes):
        x = np.random.default_rng(100 + i).integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
        dx = torch.from_numpy(x).cuda()
        dy = torch.zeros(max(n, 1), dtype=torch.int32, device="cuda")
        S.kernel_launch(0, S.make_desc(S.SCAN, n=n), [dx.data_ptr()], [dy.data_ptr()], ctas=5, stream=st.cuda_stream)
        xs.append(x)
        ys.append(dy)
    torch.cuda.synchronize()
    for x, dy in zip(xs, ys):
        y = dy.cpu().numpy().view(np.uint32)[:x.size]
        assert np.array_equal(y, K.scan(x))


def test_scan_unaligned_buffers_take_the_two_pass_body():
    torch = _torch()
    n = 3 * (1 << 20) + 11
    x = np.random.default_rng(5).integers(0, 1 << 32, n + 1, dtype=np.uint64).astype(np.uint32)
    dx = torch.from_numpy(x).cuda()
    dy = torch.zeros(n + 1, dtype=torch.int32, device="cuda")
    S.kernel_launch(0, S.make_desc(S.SCAN, n=n), [dx.data_ptr() + 4], [dy.data_ptr() + 4], ctas=37,
                    stream=torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert np.array_equal(dy.cpu().numpy().view(np.uint32)[1:], K.scan(x[1:]))


@pytest.mark.parametrize("segs", [0, 1, 3, 150, 2048])
@pytest.mark.parametrize("ctas", [0, 7])
def test_sort_bit_exact(segs, ctas):
    n = 2048 * segs
    rng = np.random.default_rng(segs)
    x = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    if n:
        x[:2048] = rng.integers(0, 4, 2048)            # many duplicates in the first segment
    (y,) = _launch(S.make_desc(S.SORT, n=n), [x], [np.zeros(n, np.uint32)], ctas)
    assert np.array_equal(y, K.sort_segments(x))


@pytest.mark.parametrize("ctas", [3, 148])
def test_sort_unaligned_pointers(ctas):
    # input and output 4 B past a 16-B boundary: the scalar load / store path of the
    # network (every group of a 4-segment round; several rounds on 3 CTAs)
    torch = _torch()
    segs = 37
    n = 2048 * segs
    x = np.random.default_rng(5).integers(0, 1 << 32, n + 1, dtype=np.uint64).astype(np.uint32)
    dx = torch.from_numpy(x.view(np.int32)).cuda()
    dy = torch.zeros(n + 1, dtype=torch.int32, device="cuda")
    S.kernel_launch(0, S.make_desc(S.SORT, n=n), [dx.data_ptr() + 4], [dy.data_ptr() + 4], ctas=ctas,
                    stream=torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert np.array_equal(dy.cpu().numpy().view(np.uint32)[1:], K.sort_segments(x[1:]))
