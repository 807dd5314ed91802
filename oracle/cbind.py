"""ctypes binding of oracle/c/kernels.c -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The plain C tenant kernels and the thread-pool job runner bench.py's
cpu_baseline leg times (plain C, -O3, no BLAS, nproc threads,
the whole workload, GEMM repeated R times).  Built with gcc on first use, or by
__graft_entry__.build().
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "c", "kernels.c")
LIB = os.path.join(HERE, "c", "liboracle_kernels.so")
CFLAGS = ["-O3", "-march=native", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-pthread"]


def build(force: bool = False) -> str:
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + ".tmp"
        subprocess.run(["gcc", *CFLAGS, SRC, "-o", tmp], check=True)
        os.replace(tmp, LIB)
    return LIB


class Job(C.Structure):
    _fields_ = [("kclass", C.c_uint32), ("reps", C.c_uint32), ("tenant", C.c_uint32), ("seed", C.c_uint32),
                ("n", C.c_uint64), ("m", C.c_uint64), ("k", C.c_uint64), ("alpha", C.c_float),
                ("in0", C.c_void_p), ("in1", C.c_void_p), ("out0", C.c_void_p)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        _lib.oc_job_struct_size.restype = C.c_uint64
        assert _lib.oc_job_struct_size() == C.sizeof(Job), "oracle/c job layout"
        _lib.oc_run_jobs.argtypes = [C.POINTER(Job), C.c_uint64, C.c_uint32]
    return _lib


def _p(a):
    return a.ctypes.data_as(C.c_void_p)


def vscale(x, a):
    x = np.ascontiguousarray(x, np.float32)
    y = np.empty_like(x)
    lib().oc_vscale(_p(x), _p(y), C.c_uint64(x.size), C.c_float(a))
    return y


def gemm(a_bits, b_bits, reps: int = 1):
    a = np.ascontiguousarray(a_bits, np.uint16)
    b = np.ascontiguousarray(b_bits, np.uint16)
    m, k = a.shape
    n = b.shape[1]
    c = np.empty((m, n), np.float32)
    lib().oc_gemm(_p(a), _p(b), _p(c), C.c_uint64(m), C.c_uint64(n), C.c_uint64(k), C.c_uint32(reps))
    return c


def xfer(x, seed):
    x = np.ascontiguousarray(x, np.uint32)
    y = np.empty_like(x)
    lib().oc_xfer(_p(x), _p(y), C.c_uint64(x.size), C.c_uint32(seed & 0xFFFFFFFF))
    return y


def hist(x):
    x = np.ascontiguousarray(x, np.uint8)
    b = np.empty(256, np.uint32)
    lib().oc_hist(_p(x), _p(b), C.c_uint64(x.size))
    return b


def scan(x):
    x = np.ascontiguousarray(x, np.uint32)
    y = np.empty_like(x)
    lib().oc_scan(_p(x), _p(y), C.c_uint64(x.size))
    return y


def sort_segments(x, seg: int = 2048):
    x = np.ascontiguousarray(x, np.uint32)
    y = np.empty_like(x)
    lib().oc_sort_segments(_p(x), _p(y), C.c_uint64(x.size), C.c_uint64(seg))
    return y


def run_jobs(specs, inputs, outputs, threads: int) -> None:
    """Every job of `specs` (strings_workload.JobSpec, submission order) on
    `threads` workers; inputs[i] / outputs[i] are numpy arrays (H2D / D2H)."""
    jobs = (Job * len(specs))()
    for i, (s, ins, outs) in enumerate(zip(specs, inputs, outputs)):
        jobs[i] = Job(kclass=s.kclass, reps=s.reps, tenant=s.tenant, seed=s.seed & 0xFFFFFFFF, n=s.n, m=s.m, k=s.k,
                      alpha=s.alpha, in0=ins[0].ctypes.data, in1=ins[1].ctypes.data if len(ins) > 1 else None,
                      out0=outs[0].ctypes.data)
    lib().oc_run_jobs(jobs, C.c_uint64(len(specs)), C.c_uint32(threads))
