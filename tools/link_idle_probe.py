"""Does the host link slow down after idling?  Times one 4 MiB (and one 256 KiB)
pinned H2D / D2H copy after the GPU's link has been idle for 0..500 ms, and right
after a 256 MiB copy, plus nvidia-smi's PCIe generation idle vs under load.

    python tools/link_idle_probe.py
"""
import json
import subprocess
import threading
import time

import torch


def smi_gen():
    try:
        out = subprocess.run(["nvidia-smi", "--query-gpu=pcie.link.gen.current,pcie.link.gen.max,"
                              "pcie.link.width.current", "--format=csv,noheader", "-i", "0"],
                             capture_output=True, text=True, timeout=20).stdout.strip()
        return out
    except Exception as e:  # noqa: BLE001
        return repr(e)


def main():
    big = 256 << 20
    hb = torch.empty(big, dtype=torch.uint8).pin_memory()
    db = torch.empty(big, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def one(sz, d2h=False):
        with torch.cuda.stream(s):
            e0.record(s)
            if d2h:
                hb[:sz].copy_(db[:sz], non_blocking=True)
            else:
                db[:sz].copy_(hb[:sz], non_blocking=True)
            e1.record(s)
        e1.synchronize()
        return e0.elapsed_time(e1) * 1e3   # us

    for _ in range(3):
        one(big)
    time.sleep(1.0)
    print(json.dumps({"smi_idle": smi_gen()}), flush=True)
    stop = []

    def load():
        while not stop:
            one(big)
    th = threading.Thread(target=load)
    th.start()
    time.sleep(0.5)
    under = smi_gen()
    stop.append(1)
    th.join()
    print(json.dumps({"smi_under_load": under}), flush=True)
    for sz in (4 << 20, 256 << 10):
        for d2h in (False, True):
            for idle_ms in (0, 1, 10, 100, 500):
                ts = []
                for _ in range(5):
                    one(big, d2h)                      # the link is busy right before
                    if idle_ms:
                        time.sleep(idle_ms / 1e3)
                    ts.append(one(sz, d2h))
                ts.sort()
                print(json.dumps({"bytes": sz, "dir": "d2h" if d2h else "h2d", "idle_ms": idle_ms,
                                  "us_median": round(ts[2], 1), "us_min": round(ts[0], 1),
                                  "us_max": round(ts[-1], 1),
                                  "GBps_median": round(sz / ts[2] / 1e3, 2)}), flush=True)
    # a burst of 16 back-to-back 4 MiB copies after 100 ms idle: per-copy times
    time.sleep(0.1)
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(17)]
    with torch.cuda.stream(s):
        evs[0].record(s)
        for i in range(16):
            db[:4 << 20].copy_(hb[:4 << 20], non_blocking=True)
            evs[i + 1].record(s)
    evs[-1].synchronize()
    print(json.dumps({"burst_after_100ms_idle_us": [round(evs[i].elapsed_time(evs[i + 1]) * 1e3, 1)
                                                   for i in range(16)]}), flush=True)


if __name__ == "__main__":
    main()
