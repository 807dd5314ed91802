"""ctypes binding of include/strings_sched.h -- argument marshalling only.

Every step of the hot path runs in libstrings_sched.so (scheduler core in C++,
tenant kernels and the persistent dispatcher in CUDA for sm_100a).  There is
no Python or CPU fallback: if the library cannot be loaded, importing this
module raises, and product timing modes return STRINGS_ECUDA without a GPU.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import List, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libstrings_sched.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "strings_sched.h")

OK, EINVAL, ENOMEM, EAGAIN, ECUDA, ESTATE, EFAULT = 0, -1, -2, -3, -4, -5, -6
VSCALE, GEMM, XFER, HIST, SCAN, SORT = 0, 1, 2, 3, 4, 5
MEASURED, INJECTED, DECISIONS_ONLY = 0, 1, 2


class StringsError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {strerror(status)} ({status})"
                         + (f", cuda error {last_cuda_error()}" if status == ECUDA else ""))


class Config(C.Structure):
    _fields_ = [("num_gpus", C.c_int32), ("physical_gpus", C.c_int32), ("balancer", C.c_int32),
                ("las_admission", C.c_int32), ("device_policy", C.c_int32), ("partitions", C.c_int32),
                ("awake_budget", C.c_int32), ("admit_cap", C.c_int32), ("joint_select", C.c_int32),
                ("timing_mode", C.c_int32), ("quantum_ns", C.c_uint64), ("slot_bytes", C.c_uint64),
                ("trace_path", C.c_char_p), ("trace_in_memory", C.c_int32),
                ("kl_mode", C.c_int32), ("reserved", C.c_int32 * 6), ("tfs_slice_ns", C.c_uint64),
                ("device_weights", C.POINTER(C.c_uint32)),
                ("ext_arenas", C.POINTER(C.c_void_p)), ("ext_arena_bytes", C.POINTER(C.c_uint64)),
                ("ext_streams", C.POINTER(C.c_void_p))]


class KernelDesc(C.Structure):
    _fields_ = [("kclass", C.c_uint32), ("reps", C.c_uint32), ("n", C.c_uint64), ("m", C.c_uint64),
                ("k", C.c_uint64), ("alpha", C.c_float), ("seed", C.c_uint32),
                ("arrival_ns", C.c_uint64), ("inj_h2d_ns", C.c_uint64), ("inj_kl_ns", C.c_uint64),
                ("inj_d2h_ns", C.c_uint64)]


class Buf(C.Structure):
    _fields_ = [("host", C.c_void_p), ("bytes", C.c_uint64)]


class JobInfo(C.Structure):
    _fields_ = [("job", C.c_uint64), ("tenant", C.c_uint32), ("seq", C.c_uint32), ("gid", C.c_int32),
                ("status", C.c_int32), ("t_arrival", C.c_uint64), ("t_place", C.c_uint64),
                ("t_start", C.c_uint64 * 3), ("t_done", C.c_uint64 * 3), ("kl_slot", C.c_int32),
                ("kl_partition", C.c_int32), ("kl_gpu_start_ns", C.c_uint64), ("kl_gpu_end_ns", C.c_uint64),
                ("kl_gpu_exec_ns", C.c_uint64), ("kl_host_issue_ns", C.c_uint64), ("kl_host_observe_ns", C.c_uint64)]


class Stats(C.Structure):
    _fields_ = [("jobs_submitted", C.c_uint64), ("jobs_done", C.c_uint64), ("jobs_failed", C.c_uint64),
                ("t_first_submit_ns", C.c_uint64), ("t_last_done_ns", C.c_uint64),
                ("h2d_bytes", C.c_uint64), ("d2h_bytes", C.c_uint64), ("kernel_bytes", C.c_uint64),
                ("kernel_flop", C.c_uint64), ("trace_records", C.c_uint64), ("decisions", C.c_uint64),
                ("decision_ns", C.c_uint64),
                ("engine_busy_ns", (C.c_uint64 * 3) * 8), ("num_gpus", C.c_int32),
                ("physical_gpus", C.c_int32), ("partitions", C.c_int32), ("sms_per_partition", C.c_int32),
                ("issue_ns", C.c_uint64), ("gpu_clock_offset_ns", C.c_int64 * 8),
                ("sm_copy_ops", C.c_uint64), ("kl_mode", C.c_int32), ("reserved_i32", C.c_int32),
                ("eager_jobs", C.c_uint64)]


def _load() -> C.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_sc_senguptagsp14_b200.build`")
    lib = C.CDLL(LIB_PATH)
    S = C.c_int32
    sig = {
        "strings_init": (S, [C.POINTER(Config)]),
        "strings_register_tenant": (S, [C.c_uint32, C.c_uint32, C.POINTER(C.c_uint32)]),
        "strings_submit": (S, [C.c_uint32, C.POINTER(KernelDesc), C.POINTER(Buf), C.c_int32,
                               C.POINTER(Buf), C.c_int32, C.c_uint32, C.POINTER(C.c_uint64)]),
        "strings_sync": (S, [C.c_uint32]),
        "strings_drain": (S, []),
        "strings_unregister_tenant": (S, [C.c_uint32]),
        "strings_shutdown": (S, []),
        "strings_host_alloc": (S, [C.c_uint64, C.POINTER(C.c_void_p)]),
        "strings_host_free": (S, [C.c_void_p]),
        "strings_job_info": (S, [C.c_uint64, C.POINTER(JobInfo)]),
        "strings_get_stats": (S, [C.POINTER(Stats)]),
        "strings_trace_size": (S, [C.POINTER(C.c_uint64)]),
        "strings_trace_copy": (S, [C.c_char_p, C.c_uint64, C.POINTER(C.c_uint64)]),
        "strings_strerror": (C.c_char_p, [S]),
        "strings_last_cuda_error": (S, []),
        "strings_version": (C.c_char_p, []),
        "strings_kernel_launch": (S, [C.c_int32, C.POINTER(KernelDesc), C.POINTER(C.c_void_p), C.c_int32,
                                      C.POINTER(C.c_void_p), C.c_int32, C.c_int32, C.c_void_p]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


lib = _load()


def declared_symbols() -> List[str]:
    """Function names declared in include/strings_sched.h."""
    import re
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"\b(strings_[a-z_]+)\s*\(", txt)) - {"strings_status_t"})


def strerror(s: int) -> str:
    return lib.strings_strerror(s).decode()


def last_cuda_error() -> int:
    return lib.strings_last_cuda_error()


def _check(s: int, where: str) -> None:
    if s != OK:
        raise StringsError(s, where)


# ------------------------------------------------------------------ calls
def init(num_gpus=0, physical_gpus=0, balancer=1, las_admission=0, device_policy=2, partitions=2,
         awake_budget=0, admit_cap=0, joint_select=-1, timing_mode=MEASURED, quantum_ns=1_000_000,
         slot_bytes=0, trace_path: Optional[str] = None, trace_in_memory=True, kl_mode=0,
         tfs_slice_ns=0, device_weights: Optional[Sequence[int]] = None,
         arenas: Optional[Sequence] = None, streams: Optional[Sequence] = None) -> None:
    """arenas: optional per-physical-GPU device buffers (torch tensors or
    (pointer, nbytes) pairs) for the resident-job slots; see torch_arenas().
    streams: optional 2 * num_gpus copy streams ([2g] H2D, [2g+1] D2H of logical
    device g): torch.cuda.Stream objects, raw cudaStream_t ints or None."""
    c = Config(num_gpus=num_gpus, physical_gpus=physical_gpus, balancer=balancer, las_admission=las_admission,
               device_policy=device_policy, partitions=partitions, awake_budget=awake_budget,
               admit_cap=admit_cap, joint_select=joint_select, timing_mode=timing_mode,
               quantum_ns=quantum_ns, slot_bytes=slot_bytes,
               trace_path=trace_path.encode() if trace_path else None,
               trace_in_memory=1 if trace_in_memory else 0, kl_mode=kl_mode, tfs_slice_ns=tfs_slice_ns)
    if device_weights is not None:
        arr = (C.c_uint32 * len(device_weights))(*device_weights)
        c.device_weights = C.cast(arr, C.POINTER(C.c_uint32))
    if arenas is not None:
        ptrs = [(a.data_ptr(), a.numel() * a.element_size()) if hasattr(a, "data_ptr") else a for a in arenas]
        pa = (C.c_void_p * len(ptrs))(*[p for p, _ in ptrs])
        pb = (C.c_uint64 * len(ptrs))(*[b for _, b in ptrs])
        c.ext_arenas = C.cast(pa, C.POINTER(C.c_void_p))
        c.ext_arena_bytes = C.cast(pb, C.POINTER(C.c_uint64))
    if streams is not None:
        hs = [0 if s is None else (s.cuda_stream if hasattr(s, "cuda_stream") else int(s)) for s in streams]
        ps = (C.c_void_p * len(hs))(*[h or None for h in hs])
        c.ext_streams = C.cast(ps, C.POINTER(C.c_void_p))
    _check(lib.strings_init(C.byref(c)), "strings_init")


def init_from_config(cfg, timing_mode=MEASURED, **kw) -> None:
    """Initialise from a strings_workload.SystemConfig (field names match)."""
    init(num_gpus=cfg.num_gpus, balancer=cfg.balancer, las_admission=cfg.las_admission,
         device_policy=cfg.device_policy, partitions=cfg.partitions, awake_budget=cfg.awake_budget,
         admit_cap=cfg.admit_cap, joint_select=cfg.joint_select, quantum_ns=cfg.quantum_ns,
         tfs_slice_ns=cfg.tfs_slice_ns, device_weights=cfg.device_weights, timing_mode=timing_mode, **kw)


DEFAULT_SLOT_BYTES = 160 << 20


def torch_arenas(num_gpus: int, physical_gpus: int, admit_cap: int, slot_bytes: int = 0):
    """Device memory for the resident-job slots allocated by PyTorch (the north
    star's "PyTorch for device memory"): one uint8 tensor per physical GPU sized
    for the logical devices mapped onto it (logical g -> physical g mod N).
    Keep the returned tensors alive until strings_shutdown."""
    import torch
    slot = slot_bytes or DEFAULT_SLOT_BYTES
    out = []
    for p in range(physical_gpus):
        n_logical = len([g for g in range(num_gpus) if g % physical_gpus == p])
        out.append(torch.empty(max(1, n_logical * admit_cap * slot), dtype=torch.uint8, device=f"cuda:{p}"))
    return out


def register_tenant(weight: int = 1, max_inflight: int = 1) -> int:
    out = C.c_uint32()
    _check(lib.strings_register_tenant(weight, max_inflight, C.byref(out)), "strings_register_tenant")
    return out.value


class HostRef:
    """A raw (address, nbytes) host buffer reference."""

    def __init__(self, addr: int, nbytes: int):
        self.addr, self.nbytes = addr, nbytes


def _addr(a) -> int:
    if isinstance(a, HostRef):
        return a.addr
    if isinstance(a, np.ndarray):
        assert a.flags["C_CONTIGUOUS"]
        return a.ctypes.data
    if hasattr(a, "data_ptr"):                      # torch tensor (pinned host)
        return a.data_ptr()
    return int(a)


def _nbytes(a) -> int:
    if isinstance(a, HostRef):
        return a.nbytes
    if isinstance(a, np.ndarray):
        return a.nbytes
    if hasattr(a, "element_size"):
        return a.numel() * a.element_size()
    raise TypeError("need numpy array or torch tensor")


def make_desc(kclass, n=0, m=0, k=0, reps=1, alpha=1.0, seed=0, arrival_ns=0, inj=(0, 0, 0)) -> KernelDesc:
    return KernelDesc(kclass=kclass, reps=reps, n=n, m=m, k=k, alpha=alpha, seed=seed & 0xFFFFFFFF,
                      arrival_ns=arrival_ns, inj_h2d_ns=inj[0], inj_kl_ns=inj[1], inj_d2h_ns=inj[2])


def submit(tenant: int, desc: KernelDesc, h2d: Sequence, d2h: Sequence, priority: int = 0) -> int:
    hb = (Buf * max(1, len(h2d)))(*[Buf(_addr(a), _nbytes(a)) for a in h2d])
    db = (Buf * max(1, len(d2h)))(*[Buf(_addr(a), _nbytes(a)) for a in d2h])
    out = C.c_uint64()
    _check(lib.strings_submit(tenant, C.byref(desc), hb, len(h2d), db, len(d2h), priority, C.byref(out)),
           "strings_submit")
    return out.value


def submit_spec(tenant: int, spec, h2d: Sequence, d2h: Sequence) -> int:
    """Submit a strings_workload.JobSpec."""
    desc = make_desc(spec.kclass, n=spec.n, m=spec.m, k=spec.k, reps=spec.reps, alpha=spec.alpha,
                     seed=spec.seed, arrival_ns=spec.arrival_ns,
                     inj=(spec.inj_h2d_ns, spec.inj_kl_ns, spec.inj_d2h_ns))
    return submit(tenant, desc, h2d, d2h, spec.priority)


def sync(tenant: int) -> int:
    return lib.strings_sync(tenant)


def drain() -> int:
    return lib.strings_drain()


def unregister_tenant(tenant: int) -> int:
    return lib.strings_unregister_tenant(tenant)


def shutdown() -> int:
    return lib.strings_shutdown()


def host_alloc(nbytes: int) -> int:
    p = C.c_void_p()
    _check(lib.strings_host_alloc(nbytes, C.byref(p)), "strings_host_alloc")
    return p.value


def host_free(p: int) -> None:
    _check(lib.strings_host_free(p), "strings_host_free")


def pinned_array(shape, dtype) -> np.ndarray:
    """A numpy view on library-pinned host memory (zero-copy fast path).  The
    memory is released by free_pinned(arr)."""
    dtype = np.dtype(dtype)
    n = int(np.prod(shape)) * dtype.itemsize
    p = host_alloc(max(1, n))
    buf = (C.c_uint8 * max(1, n)).from_address(p)
    a = np.frombuffer(buf, dtype=np.uint8, count=n).view(dtype).reshape(shape)
    _PINNED[id(a)] = p
    return a


_PINNED = {}


def free_pinned(a: np.ndarray) -> None:
    p = _PINNED.pop(id(a), None)
    if p is not None:
        host_free(p)


def job_info(job: int) -> JobInfo:
    info = JobInfo()
    _check(lib.strings_job_info(job, C.byref(info)), "strings_job_info")
    return info


def stats() -> Stats:
    s = Stats()
    _check(lib.strings_get_stats(C.byref(s)), "strings_get_stats")
    return s


def trace() -> List[str]:
    n = C.c_uint64()
    _check(lib.strings_trace_size(C.byref(n)), "strings_trace_size")
    buf = C.create_string_buffer(n.value + 1)
    w = C.c_uint64()
    lib.strings_trace_copy(buf, n.value, C.byref(w))
    return buf.raw[: w.value].decode().splitlines()


def kernel_launch(gpu: int, desc: KernelDesc, dev_in: Sequence[int], dev_out: Sequence[int], ctas: int = 0,
                  stream: int = 0) -> None:
    ins = (C.c_void_p * len(dev_in))(*dev_in)
    outs = (C.c_void_p * len(dev_out))(*dev_out)
    _check(lib.strings_kernel_launch(gpu, C.byref(desc), ins, len(dev_in), outs, len(dev_out), ctas,
                                     C.c_void_p(stream)), "strings_kernel_launch")


def version() -> str:
    return lib.strings_version().decode()
