"""Host-link rate by pinned-allocation method: torch pin_memory vs the library's
strings_host_alloc (cudaHostAlloc portable|mapped), for 4 MiB and 64 MiB copies.

    python tools/pinned_alloc_probe.py
"""
import ctypes
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402

MiB = 1 << 20


def main():
    out = []
    for size in (256 << 10, 4 * MiB, 64 * MiB):
        bufs = {
            "torch_pin_memory": (torch.empty(size, dtype=torch.uint8).pin_memory(),
                                 torch.empty(size, dtype=torch.uint8).pin_memory()),
        }
        a = S.pinned_array((size,), np.uint8)
        b = S.pinned_array((size,), np.uint8)
        a[...] = 1
        b[...] = 2
        bufs["strings_host_alloc"] = (torch.from_numpy(a), torch.from_numpy(b))
        dev_in = torch.empty(size, dtype=torch.uint8, device="cuda")
        dev_out = torch.empty(size, dtype=torch.uint8, device="cuda")
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        reps = max(4, (256 * MiB) // size)
        for name, (hi, ho) in bufs.items():
            res = {"alloc": name, "bytes": size}
            for mode in ("h2d", "d2h", "bidir"):
                best = None
                for _ in range(3):
                    torch.cuda.synchronize()
                    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                    e0.record(s1)
                    s2.wait_event(e0)
                    if mode in ("h2d", "bidir"):
                        with torch.cuda.stream(s1):
                            for _ in range(reps):
                                dev_in.copy_(hi, non_blocking=True)
                    if mode in ("d2h", "bidir"):
                        with torch.cuda.stream(s2):
                            for _ in range(reps):
                                ho.copy_(dev_out, non_blocking=True)
                    e1.record(s1)
                    e2.record(s2)
                    torch.cuda.synchronize()
                    dt = max(e0.elapsed_time(e1), e0.elapsed_time(e2)) / 1e3
                    best = dt if best is None else min(best, dt)
                res[f"{mode}_GBps_per_dir"] = round(size * reps / best / 1e9, 2)
            # a lone copy after a pause
            lone = []
            for _ in range(5):
                torch.cuda.synchronize()
                time.sleep(0.002)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s1)
                with torch.cuda.stream(s1):
                    dev_in.copy_(hi, non_blocking=True)
                e1.record(s1)
                torch.cuda.synchronize()
                lone.append(e0.elapsed_time(e1) * 1e3)
            res["lone_h2d_us_min"] = round(min(lone), 1)
            print(json.dumps(res), flush=True)
            out.append(res)


if __name__ == "__main__":
    main()
