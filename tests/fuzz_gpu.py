"""Extended GPU fuzz (not part of the test tier): random workloads in MEASURED and
INJECTED timing through the library (copy partition, busy policy, KL partitions),
each checked against the oracle (INJECTED trace byte-identical, MEASURED
invariants) and every output against the oracle's CPU kernels.

    python tests/fuzz_gpu.py [first_seed] [count] [big]   (test infrastructure: it runs the oracle)

`big`: BASELINE-sized VSCALE / XFER jobs (4 / 64 MiB), so MEASURED runs take the
eager chaining path when its condition holds.  Every run draws the issuer-thread
mode (STRINGS_ISSUE_THREADS) from the seed.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import strings_workload as W  # noqa: E402
from oracle import invariants  # noqa: E402
from oracle.des import run_oracle  # noqa: E402
from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402
from paper_conf_sc_senguptagsp14_b200.runner import run_workload  # noqa: E402
from test_gpu_scheduler import check_outputs  # noqa: E402


def main():
    first = int(sys.argv[1]) if len(sys.argv) > 1 else 1000
    count = int(sys.argv[2]) if len(sys.argv) > 2 else 100
    big = len(sys.argv) > 3 and sys.argv[3] == "big"
    bad = eager = 0
    for seed in range(first, first + count):
        wl = W.random_workload(seed, max_gpus=3, tiny=not big)
        for timing in (S.MEASURED, S.INJECTED):
            os.environ["STRINGS_ISSUE_THREADS"] = str((seed + timing) % 2)
            try:
                r = run_workload(wl, timing_mode=timing)
                assert r.status == S.OK, r.status
                if timing == S.INJECTED:
                    assert r.trace == run_oracle(wl).trace, "trace differs"
                else:
                    errs = invariants.check(r.trace, wl)
                    assert errs == [], errs[:3]
                check_outputs(wl, r)
                eager += r.stats.eager_jobs
            except AssertionError as e:
                bad += 1
                print(f"seed {seed} timing {timing}: FAIL {str(e)[:200]}", flush=True)
    print(f"fuzz: {count} workloads x 2 timings ({'big' if big else 'tiny'}), {eager} eager jobs, {bad} failures",
          flush=True)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
