"""Scheduler overhead per job on an idle B200 (SURVEY §8(d) "the scheduler's own work").

One tenant submits tiny jobs one at a time (VSCALE n=1024: 4 KB each way) and
syncs after each; the library's job records give host-observed phase times and
the dispatcher's %globaltimer stamps.  Reported medians (us):
  h2d / kl / d2h  host-observed START->DONE per phase
  kl_device       device claim -> last CTA done (the KL body itself + broadcast)
  submit_to_done  strings_submit -> JOB_DONE (library clock)
  sync_rtt        Python submit() call -> sync() return (wall clock)
"""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402


def main(n_jobs=300, n=1024):
    S.init(num_gpus=1, physical_gpus=1, timing_mode=S.MEASURED, balancer=1, device_policy=2)
    try:
        t = S.register_tenant(1, 1)
        x = S.pinned_array((n,), np.float32)
        y = S.pinned_array((n,), np.float32)
        x[:] = 1.5
        rtt = []
        for i in range(n_jobs):
            t0 = time.perf_counter()
            S.submit(t, S.make_desc(S.VSCALE, n=n, alpha=2.0), [x], [y])
            assert S.sync(t) == S.OK
            rtt.append((time.perf_counter() - t0) * 1e6)
        assert float(y[0]) == 3.0
        infos = [S.job_info(i) for i in range(n_jobs)][20:]
        off = S.stats().gpu_clock_offset_ns[0]
    finally:
        S.shutdown()
    med = lambda v: round(statistics.median(v), 2)
    out = {
        "jobs": n_jobs - 20, "bytes_each_way": 4 * n,
        "h2d_us": med([(i.t_done[0] - i.t_start[0]) / 1e3 for i in infos]),
        "kl_us": med([(i.t_done[1] - i.t_start[1]) / 1e3 for i in infos]),
        "d2h_us": med([(i.t_done[2] - i.t_start[2]) / 1e3 for i in infos]),
        "kl_device_us": med([(i.kl_gpu_end_ns - i.kl_gpu_start_ns) / 1e3 for i in infos]),
        "submit_to_done_us": med([(i.t_done[2] - i.t_arrival) / 1e3 for i in infos]),
        "sync_rtt_us": med(rtt[20:]),
        # decomposition of the KL phase: device %globaltimer stamps moved onto the host
        # CLOCK_REALTIME line with the offset the library calibrates at init (+-RTT/2)
        "gpu_clock_offset_ns": off,
        "kl_issue_to_claim_us": med([(i.kl_gpu_start_ns - off - i.kl_host_issue_ns) / 1e3 for i in infos]),
        "kl_claim_to_exec_us": med([(i.kl_gpu_exec_ns - i.kl_gpu_start_ns) / 1e3 for i in infos]),
        "kl_exec_to_end_us": med([(i.kl_gpu_end_ns - i.kl_gpu_exec_ns) / 1e3 for i in infos]),
        "kl_end_to_observe_us": med([(i.kl_host_observe_ns - (i.kl_gpu_end_ns - off)) / 1e3 for i in infos]),
        "kl_issue_to_observe_us": med([(i.kl_host_observe_ns - i.kl_host_issue_ns) / 1e3 for i in infos]),
    }
    print(json.dumps(out))


if __name__ == "__main__":
    main()
