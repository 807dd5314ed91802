"""HBM ceiling of an SM partition: XFER / VSCALE bodies stand-alone on `ctas`
CTAs (CUDA events, 20 launches, 2^24 elements = 128 MiB moved, > L2 when
rotating 4 buffer pairs), alone and with two partitions running at once on
two streams.  The dispatcher's XFER item (C2: 74-SM partition) is judged
against this ceiling.

    python tools/partition_probe.py
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402


def main():
    n = 1 << 24
    nb = 4
    xs = [torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda") for _ in range(2 * nb)]
    ys = [torch.empty_like(x) for x in xs]
    s0, s1 = torch.cuda.Stream(), torch.cuda.Stream()
    kinds = ((S.XFER, "XFER"), (S.VSCALE, "VSCALE"))
    if os.environ.get("PROBE_QUICK"):
        kinds = kinds[:1]
    for cls, name in kinds:
        desc = S.make_desc(cls, n=n, alpha=1.001, seed=7)
        for ctas in ((37, 74, 148) if os.environ.get("PROBE_QUICK") else (18, 37, 74, 111, 148)):
            for pair in (False, True):
                if pair and ctas > 74:
                    continue
                iters = 20
                for _ in range(2):
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(s0)
                    s1.wait_event(e0)
                    for i in range(iters):
                        b = i % nb
                        S.kernel_launch(0, desc, [xs[b].data_ptr()], [ys[b].data_ptr()], ctas=ctas,
                                        stream=s0.cuda_stream)
                        if pair:
                            S.kernel_launch(0, desc, [xs[nb + b].data_ptr()], [ys[nb + b].data_ptr()], ctas=ctas,
                                            stream=s1.cuda_stream)
                    e = torch.cuda.Event()
                    e.record(s1)
                    s0.wait_event(e)
                    e1.record(s0)
                    torch.cuda.synchronize()
                    ms = e0.elapsed_time(e1)
                moved = 8 * n * iters * (2 if pair else 1)
                print(json.dumps({"variant": os.environ.get("STRINGS_NVCC_EXTRA", ""), "kernel": name, "ctas": ctas, "partitions": 2 if pair else 1,
                                  "us_per_launch": round(ms * 1e3 / iters, 2),
                                  "GBps_total": round(moved / ms / 1e6, 1),
                                  "GBps_per_partition": round(moved / ms / 1e6 / (2 if pair else 1), 1)}), flush=True)


if __name__ == "__main__":
    main()
