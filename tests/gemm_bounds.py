"""Element-wise error bound for the tensor-core GEMM (test helper, no GPU needed)."""
import numpy as np

from oracle import kernels as K


def gemm_elementwise_ok(c, a_bits, b_bits):
    """Element-wise bound for C = A.B with bf16 operands and fp32 accumulation
    (reading R-22): every bf16 x bf16 product is exact in fp32, and the tensor
    core adds K/16 partial sums of 16 products into the fp32 accumulator, each
    addition rounding once, so |c - r| <= (K/16 + 1) * u * sum_k |a_ik b_kj|
    plus one final rounding of r itself (u |r|), with u = 2^-23: twice fp32's
    unit roundoff, allowing the MMA's internal alignment to truncate instead of
    rounding to nearest.  Checked beside the normwise 1e-5 of R-22."""
    a = K.bf16_bits_to_f64(a_bits)
    b = K.bf16_bits_to_f64(b_bits)
    r = a @ b
    mag = np.abs(a) @ np.abs(b)
    k = a.shape[1]
    u = 2.0 ** -23
    bound = (k / 16 + 1) * u * mag + u * np.abs(r)
    return bool(np.all(np.abs(c.astype(np.float64) - r) <= bound))
