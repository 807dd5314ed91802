"""Plain pre-queued copy replay of a config's buffers vs the number of copy
streams per direction (bench.copy_replay_s), plus synthetic uniform-size mixes.

    python tools/replay_probe.py
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
import strings_workload as W  # noqa: E402


class _Job:
    def __init__(self, h, d):
        self._h, self._d = h, d

    def h2d_sizes(self):
        return self._h

    def d2h_sizes(self):
        return self._d


class _Wl:
    def __init__(self, jobs):
        self.jobs = jobs


def main():
    cases = {name: W.CONFIGS[name]() for name in ("C1", "C3")}
    cases["4MiB x128"] = _Wl([_Job([4 << 20], [4 << 20]) for _ in range(128)])
    cases["4MiB x128 h2d only"] = _Wl([_Job([4 << 20], []) for _ in range(128)])
    cases["128KiB x512"] = _Wl([_Job([128 << 10], [128 << 10]) for _ in range(512)])
    for name, wl in cases.items():
        hb = sum(sum(j.h2d_sizes()) for j in wl.jobs)
        db = sum(sum(j.d2h_sizes()) for j in wl.jobs)
        row = {"case": name, "h2d_MiB": hb >> 20, "d2h_MiB": db >> 20}
        for s in (1, 2, 4, 8):
            t = bench.copy_replay_s(torch, wl, s, reps=3)
            row[f"s{s}_ms"] = round(t * 1e3, 3)
            row[f"s{s}_GBps_per_dir"] = round(max(hb, db) / t / 1e9, 2)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
