"""Pins for oracle/kernels.py against things other than itself (no GPU)."""
import math
import struct

import numpy as np
import pytest

import strings_workload as W
from oracle import kernels as K


# --------------------------------------------------------------------- VSCALE
def _f32(v):
    try:
        return struct.unpack("<f", struct.pack("<f", v))[0]
    except OverflowError:            # rounds beyond FLT_MAX -> +-inf under RNE
        return math.copysign(math.inf, v)


def test_vscale_is_correctly_rounded_product():
    # fp32 x fp32 is exact in fp64 (24+24 < 53 bits); one rounding to fp32
    # (struct 'f' packing rounds to nearest-even) is the IEEE product.
    rng = np.random.default_rng(7)
    x = np.concatenate([
        rng.uniform(-1, 1, 5000).astype(np.float32),
        np.array([0.0, -0.0, 1e-45, -1e-45, 1.17549435e-38, 3.4028235e38, -3.4028235e38,
                  1.5e-39, 2.0 ** -130], dtype=np.float32)])
    for alpha in (1.0 + 2.0 ** -10, -0.3333333, 2.0 ** -20, 3.0e10):
        got = K.vscale(x, alpha)
        a32 = _f32(alpha)
        want = np.array([_f32(float(v) * a32) for v in x.tolist()], dtype=np.float32)
        assert got.dtype == np.float32
        assert np.array_equal(got.view(np.uint32), want.view(np.uint32))


def test_vscale_denormals_preserved():
    x = np.array([2.0 ** -126], dtype=np.float32)
    y = K.vscale(x, 0.5)
    assert y[0] == np.float32(2.0 ** -127) and y[0] != 0


# ----------------------------------------------------------------------- GEMM
def test_bf16_widening_known_values():
    bits = np.array([0x3F80, 0xC000, 0x0000, 0x8000, 0x3EAB, 0x7F7F], dtype=np.uint16)
    v = K.bf16_bits_to_f64(bits)
    assert v[0] == 1.0 and v[1] == -2.0 and v[2] == 0.0 and math.copysign(1, v[3]) == -1
    assert v[4] == 0.333984375                      # 0x3EAB = 1.3359375 * 2^-2
    assert v[5] == 3.3895313892515355e38            # largest finite bf16


def test_bf16_rounding_of_generator_is_rne():
    x = np.array([1.0, 1.00390625, 1.01171875, 1.0 + 2 ** -9, -1.0 - 3 * 2 ** -9], dtype=np.float32)
    b = W.f32_to_bf16_bits(x)
    # 1+2^-8 ties 1 vs 1+2^-7 -> even (1.0); 1+3*2^-8 ties -> 1+2^-6 (even);
    # 1+2^-9 is 1/4 ulp -> 1.0; -(1+3*2^-9) is 3/4 ulp -> -(1+2^-7)
    assert b.tolist() == [0x3F80, 0x3F80, 0x3F82, 0x3F80, 0xBF81]


def test_gemm_integer_inputs_exact_vs_int64_triple_loop():
    rng = np.random.default_rng(3)
    m, n, k = 16, 24, 40
    ai = rng.integers(-2, 3, size=(m, k))
    bi = rng.integers(-2, 3, size=(k, n))
    a = W.f32_to_bf16_bits(ai.astype(np.float32))
    b = W.f32_to_bf16_bits(bi.astype(np.float32))
    c = K.gemm(a, b)
    want = np.zeros((m, n), dtype=np.int64)
    for i in range(m):
        for j in range(n):
            s = 0
            for t in range(k):
                s += int(ai[i, t]) * int(bi[t, j])
            want[i, j] = s
    assert np.array_equal(c, want.astype(np.float32))


def test_gemm_random_within_one_ulp_of_exact_sum():
    rng = np.random.default_rng(11)
    m, n, k = 8, 8, 256
    a = W.f32_to_bf16_bits(rng.uniform(-1, 1, (m, k)).astype(np.float32))
    b = W.f32_to_bf16_bits(rng.uniform(-1, 1, (k, n)).astype(np.float32))
    c = K.gemm(a, b)
    av, bv = K.bf16_bits_to_f64(a), K.bf16_bits_to_f64(b)
    for i in range(m):
        for j in range(n):
            exact = math.fsum(float(av[i, t]) * float(bv[t, j]) for t in range(k))  # bf16*bf16 exact in fp64
            r = np.float32(exact)
            assert abs(float(c[i, j]) - float(r)) <= float(np.spacing(np.abs(r)))


def test_gemm_transposition_sensitive():
    # A.B != B.A for a non-symmetric case: catches a transposed operand
    a = W.f32_to_bf16_bits(np.array([[1, 2], [0, 1]], dtype=np.float32))
    b = W.f32_to_bf16_bits(np.array([[1, 0], [3, 1]], dtype=np.float32))
    assert K.gemm(a, b).tolist() == [[7.0, 2.0], [3.0, 1.0]]


# ----------------------------------------------------------------------- XFER
def test_fmix32_published_murmur3_vectors():
    # MurmurHash3_x86_32 of the empty key is fmix32(seed ^ 0):
    #   ("", 0) -> 0, ("", 1) -> 0x514E28B7, ("", 0xFFFFFFFF) -> 0x81F16F39
    # and of "\0\0\0\0" with seed 0 the body leaves h = 0xE6546B64, ^len -> 0xE6546B60,
    #   hash = 0x2362F9DE   (SMHasher verification vectors).
    x = np.array([0, 1, 0xFFFFFFFF, 0xE6546B60], dtype=np.uint32)
    assert K.fmix32(x).tolist() == [0, 0x514E28B7, 0x81F16F39, 0x2362F9DE]


def test_xfer_is_fmix_of_xor_and_bijective_sample():
    x = np.arange(1 << 16, dtype=np.uint32)
    y = K.xfer(x, 1)
    assert y[0] == 0x514E28B7                 # fmix32(0 ^ 1)
    assert len(np.unique(y)) == len(y)        # a bijection has no collisions


@pytest.mark.parametrize("cls", [W.VSCALE, W.GEMM, W.XFER])
def test_run_job_shapes(cls):
    j = {W.VSCALE: W.JobSpec(0, W.VSCALE, n=1000, alpha=2.0, data_seed=1),
         W.GEMM: W.JobSpec(0, W.GEMM, m=128, n=256, k=64, data_seed=2),
         W.XFER: W.JobSpec(0, W.XFER, n=1000, seed=5, data_seed=3)}[cls]
    ins = W.job_inputs(j)
    assert [a.nbytes for a in ins] == j.h2d_sizes()
    outs = K.run_job(j, ins)
    assert [a.nbytes for a in outs] == j.d2h_sizes()


# ------------------------------------------------- NEXT-2 (Table I shapes)
def test_hist_brute_force_and_total():
    rng = np.random.default_rng(5)
    x = rng.integers(0, 256, 3000).astype(np.uint8)
    h = K.hist(x)
    want = [0] * 256
    for v in x.tolist():
        want[v] += 1
    assert h.tolist() == want and h.dtype == np.uint32 and int(h.sum()) == x.size
    assert K.hist(np.zeros(0, np.uint8)).tolist() == [0] * 256


def test_scan_definition_wraps_mod_2_32():
    x = np.array([0xFFFFFFFF, 2, 3, 0x80000000, 0x80000000], dtype=np.uint32)
    acc, want = 0, []
    for v in x.tolist():
        acc = (acc + v) % (1 << 32)
        want.append(acc)
    assert K.scan(x).tolist() == want
    rng = np.random.default_rng(1)
    y = rng.integers(0, 1 << 32, 10000, dtype=np.uint64).astype(np.uint32)
    s = K.scan(y)
    assert s[0] == y[0] and np.array_equal((s[1:] - s[:-1]).astype(np.uint32), y[1:])   # difference invariant


def test_sort_segments_sorted_permutation():
    rng = np.random.default_rng(2)
    x = rng.integers(0, 1 << 32, 3 * 2048, dtype=np.uint64).astype(np.uint32)
    y = K.sort_segments(x)
    for sgm in range(3):
        a, b = x[sgm * 2048:(sgm + 1) * 2048], y[sgm * 2048:(sgm + 1) * 2048]
        assert np.all(b[1:] >= b[:-1])                        # ascending
        assert sorted(a.tolist()) == b.tolist()               # a permutation of its own segment
    assert K.sort_segments(np.array([3, 1, 2, 0], np.uint32), seg=4).tolist() == [0, 1, 2, 3]


def test_gemm_elementwise_bound_accepts_fp32_accumulation_and_rejects_errors():
    # the GPU tests' element-wise GEMM bound (tests/gemm_bounds.py, R-22): a plain
    # sequential fp32 accumulation of the exact bf16 products stays inside it; a
    # result rounded to bf16, or one with a single wrong product, does not
    from gemm_bounds import gemm_elementwise_ok
    rng = np.random.default_rng(5)
    a = W.f32_to_bf16_bits(rng.uniform(-1, 1, (128, 256)).astype(np.float32))
    b = W.f32_to_bf16_bits(rng.uniform(-1, 1, (256, 256)).astype(np.float32))
    af, bf = K.bf16_bits_to_f64(a).astype(np.float32), K.bf16_bits_to_f64(b).astype(np.float32)
    c = np.zeros((128, 256), np.float32)
    for kk in range(256):
        c += af[:, kk:kk + 1] * bf[kk:kk + 1, :]
    assert gemm_elementwise_ok(c, a, b)
    assert not gemm_elementwise_ok(K.bf16_bits_to_f64(W.f32_to_bf16_bits(c)).astype(np.float32), a, b)
    bad = c.copy()
    bad[3, 7] += af[3, 11] * bf[11, 7]           # one product counted twice
    assert not gemm_elementwise_ok(bad, a, b)
