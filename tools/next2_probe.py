"""NEXT-2 tenant kernels stand-alone on the whole GPU (HIST, SCAN, SORT), CUDA-event
timed, inputs larger than L2: achieved GB/s of algorithmic bytes vs the HBM peak.

    python tools/next2_probe.py
HIST: n bytes in, 256 u32 bins out (n + 1 KiB); SCAN: n u32 in and out (8n);
SORT: 2048-key segments, n u32 in and out (8n; bitonic network in shared memory).
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402


def main():
    peaks = bench.measured_peaks()
    st = torch.cuda.current_stream()

    def timed(desc, ins, outs, iters=10, ctas=0):
        S.kernel_launch(0, desc, [a.data_ptr() for a in ins], [a.data_ptr() for a in outs], ctas=ctas,
                        stream=st.cuda_stream)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(iters):
            S.kernel_launch(0, desc, [a.data_ptr() for a in ins], [a.data_ptr() for a in outs], ctas=ctas,
                            stream=st.cuda_stream)
        e1.record(st)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / 1e3 / iters

    n = 1 << 30
    x = torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda")
    h = torch.zeros(256, dtype=torch.int32, device="cuda")
    t = timed(S.make_desc(S.HIST, n=n), [x], [h])
    rows = [("HIST", n + 1024, t, f"n=2^30 bytes")]
    del x
    # the pairwise mix's HIST job (2^26 image-like bytes) on all SMs and on one 72-SM KL
    # slot; 8 rotating inputs (512 MiB > L2)
    import strings_workload as W
    xs = [torch.from_numpy(W.job_inputs(W.JobSpec(tenant=0, kclass=W.HIST, n=1 << 26, data_seed=s))[0]).cuda()
          for s in range(8)]
    for ctas in (0, 72):
        ts = [timed(S.make_desc(S.HIST, n=1 << 26), [xs[i]], [h], iters=4, ctas=ctas) for i in range(8)]
        rows.append(("HIST", (1 << 26) + 1024, sum(ts) / len(ts), f"n=2^26 image-like bytes, {ctas or 'all'} CTAs"))
    assert torch.equal(h.long(), torch.bincount(xs[7].long(), minlength=256))
    del xs
    n = 1 << 28
    x = torch.randint(0, 1 << 20, (n,), dtype=torch.int32, device="cuda")
    y = torch.empty_like(x)
    rows.append(("SCAN", 8 * n, timed(S.make_desc(S.SCAN, n=n), [x], [y]), "n=2^28 u32"))
    rows.append(("SORT", 8 * n, timed(S.make_desc(S.SORT, n=n), [x], [y]), "n=2^28 u32, 2048-key segments"))
    for name, b, t, size in rows:
        g = b / t / 1e9
        print(json.dumps({"kernel": name, "size": size, "bytes": b, "ms": round(t * 1e3, 4), "achieved_GBps": round(g, 1),
                          "hbm_peak": peaks["hbm_gbs"], "frac": round(g / peaks["hbm_gbs"], 4)}), flush=True)


if __name__ == "__main__":
    main()
