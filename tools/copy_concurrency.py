"""Aggregate host-link bandwidth vs the number of concurrent copy streams.

N streams each copy `--mib` MiB (pinned host <-> device, separate buffers per
stream), all issued at once; aggregate GB/s = total bytes / (last done - first
issue).  Directions: h2d, d2h, and both (N H2D + N D2H streams).

    python tools/copy_concurrency.py [--mib 64] [--reps 3]
"""
import argparse
import json
import time

import torch


def run(n, mib, direction, reps):
    nb = mib << 20
    hs = [torch.empty(nb, dtype=torch.uint8).pin_memory() for _ in range(n)]
    ds = [torch.empty(nb, dtype=torch.uint8, device="cuda") for _ in range(n)]
    hs2 = [torch.empty(nb, dtype=torch.uint8).pin_memory() for _ in range(n)] if direction == "both" else []
    ds2 = [torch.empty(nb, dtype=torch.uint8, device="cuda") for _ in range(n)] if direction == "both" else []
    st = [torch.cuda.Stream() for _ in range(n)]
    st2 = [torch.cuda.Stream() for _ in range(n)] if direction == "both" else []
    best = None
    for _ in range(reps + 1):
        torch.cuda.synchronize()
        t = time.perf_counter()
        for i in range(n):
            with torch.cuda.stream(st[i]):
                if direction in ("h2d", "both"):
                    ds[i].copy_(hs[i], non_blocking=True)
                else:
                    hs[i].copy_(ds[i], non_blocking=True)
            if direction == "both":
                with torch.cuda.stream(st2[i]):
                    hs2[i].copy_(ds2[i], non_blocking=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t
        best = dt if best is None else min(best, dt)
    total = n * nb * (2 if direction == "both" else 1)
    return total / best / 1e9


def run_serial(k, kib, reps):
    """k back-to-back copies of `kib` KiB on ONE stream (DMA pipelining)."""
    nb = kib << 10
    hs = [torch.empty(nb, dtype=torch.uint8).pin_memory() for _ in range(k)]
    ds = [torch.empty(nb, dtype=torch.uint8, device="cuda") for _ in range(k)]
    st = torch.cuda.Stream()
    best = None
    for _ in range(reps + 1):
        torch.cuda.synchronize()
        t = time.perf_counter()
        with torch.cuda.stream(st):
            for i in range(k):
                ds[i].copy_(hs[i], non_blocking=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t
        best = dt if best is None else min(best, dt)
    return k * nb / best / 1e9


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--mib", type=int, nargs="*", default=[64, 4])
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    for mib in args.mib:
        for direction in ("h2d", "d2h", "both"):
            row = {"direction": direction, "mib_per_copy": mib}
            for n in (1, 2, 4, 8, 16):
                row[f"n{n}_GBps"] = round(run(n, mib, direction, args.reps), 2)
                torch.cuda.empty_cache()
            print(json.dumps(row), flush=True)
    for kib in (256, 4096):
        row = {"direction": "h2d one stream, k back-to-back copies", "kib_per_copy": kib}
        for k in (1, 2, 4, 16):
            row[f"k{k}_GBps"] = round(run_serial(k, kib, args.reps), 2)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
