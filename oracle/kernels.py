"""Plain CPU definitions of the three tenant kernel classes.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  These are the closed-form
results the CUDA tenant kernels must reproduce (SURVEY.md §8(c) "Plain CPU
kernels"; the paper's workload classes, Table I):

* VSCALE -- streaming memory-bound:  y[i] = a * x[i], one IEEE fp32 multiply,
  round-to-nearest-even, no FMA, denormals preserved (reading R-23).  Bit-exact.
* GEMM   -- compute-bound dense:    C = A . B with A (m x k), B (k x n) bf16
  row-major, products and sums in fp64, rounded once to fp32 (reading R-22).
  The KL phase repeats the product R times; every repetition yields the same C,
  so R does not enter the result.
* XFER   -- transfer-heavy:          y[i] = fmix32(x[i] ^ seed) in uint32, the
  MurmurHash3 finaliser (reading R-17).  Bit-exact.

NEXT-2 classes shaped like the paper's Table I applications:
* HIST   -- Histogram (HI):   bins[b] = #{i : x[i] == b}, 256 bins, uint32.
* SCAN   -- Scan (SC):        y[i] = x[0] + ... + x[i]  mod 2^32 (inclusive).
* SORT   -- Sorting Networks (SN): every consecutive 2048-key segment sorted
  ascending (the SDK sample sorts a batch of fixed-length arrays).
All three are bit-exact.
"""
from __future__ import annotations

import numpy as np


def bf16_bits_to_f64(bits: np.ndarray) -> np.ndarray:
    """bf16 bit pattern -> exact float64 value (a bf16 is the top half of an fp32)."""
    f32 = (np.asarray(bits, dtype=np.uint16).astype(np.uint32) << 16).view(np.float32)
    return f32.astype(np.float64)


def vscale(x: np.ndarray, alpha: float) -> np.ndarray:
    """y = alpha * x, single fp32 multiply per element."""
    x = np.asarray(x, dtype=np.float32)
    return np.multiply(x, np.float32(alpha), dtype=np.float32)


def gemm(a_bits: np.ndarray, b_bits: np.ndarray) -> np.ndarray:
    """C = A . B: widen bf16 -> fp64, fp64 matrix product, one rounding to fp32."""
    a = bf16_bits_to_f64(a_bits)
    b = bf16_bits_to_f64(b_bits)
    return (a @ b).astype(np.float32)


def fmix32(h: np.ndarray) -> np.ndarray:
    """MurmurHash3 32-bit finaliser (Appleby), uint32 wrap-around arithmetic."""
    h = np.asarray(h, dtype=np.uint32).copy()
    h ^= h >> np.uint32(16)
    h *= np.uint32(0x85EBCA6B)
    h ^= h >> np.uint32(13)
    h *= np.uint32(0xC2B2AE35)
    h ^= h >> np.uint32(16)
    return h


def xfer(x: np.ndarray, seed: int) -> np.ndarray:
    """y = fmix32(x ^ seed)."""
    return fmix32(np.asarray(x, dtype=np.uint32) ^ np.uint32(seed & 0xFFFFFFFF))


def hist(x: np.ndarray) -> np.ndarray:
    """256-bin byte histogram (counts fit uint32 for n < 2^32)."""
    return np.bincount(np.asarray(x, dtype=np.uint8), minlength=256).astype(np.uint32)


def scan(x: np.ndarray) -> np.ndarray:
    """Inclusive prefix sum modulo 2^32 (uint32 wrap-around)."""
    return np.cumsum(np.asarray(x, dtype=np.uint32), dtype=np.uint32)


def sort_segments(x: np.ndarray, seg: int = 2048) -> np.ndarray:
    """Each consecutive segment of `seg` keys sorted ascending."""
    x = np.asarray(x, dtype=np.uint32)
    assert x.size % seg == 0
    return np.sort(x.reshape(-1, seg), axis=1).reshape(-1)


def run_job(spec, inputs):
    """Outputs (list of arrays) of one job given its H2D inputs."""
    import strings_workload as W
    if spec.kclass == W.VSCALE:
        return [vscale(inputs[0], spec.alpha)]
    if spec.kclass == W.GEMM:
        return [gemm(inputs[0].reshape(spec.m, spec.k), inputs[1].reshape(spec.k, spec.n))]
    if spec.kclass == W.XFER:
        return [xfer(inputs[0], spec.seed)]
    if spec.kclass == W.HIST:
        return [hist(inputs[0])]
    if spec.kclass == W.SCAN:
        return [scan(inputs[0])]
    if spec.kclass == W.SORT:
        return [sort_segments(inputs[0], W.SORT_SEGMENT)]
    raise ValueError(spec.kclass)
