"""How fast are single, dependent 4 MiB copies when both directions are busy?
(C1's VSCALE chains: each tenant H2D -> (KL) -> D2H -> next H2D, c_t = 1.)

    python tools/chain_probe.py

Cases (pinned buffers per tenant, device-timed with events, no kernels):
  single_h2d / single_d2h: one 4 MiB copy alone on an idle link
  pair_bidir: one H2D and one D2H issued together on two streams
  prequeued_bidir: 16 H2D + 16 D2H pre-queued (two streams)
  chains2: two tenants, each chain H2D -> D2H -> H2D ... (8 jobs) on its own
           stream pair with event dependencies, so at most one copy per
           tenant is in flight, as under the scheduler with c_t = 1
"""
import json
import time

import torch

MiB = 1 << 20


def ev():
    return torch.cuda.Event(enable_timing=True)


def main():
    n = 4 * MiB
    T = 2
    hin = [torch.empty(n, dtype=torch.uint8).pin_memory() for _ in range(T)]
    hout = [torch.empty(n, dtype=torch.uint8).pin_memory() for _ in range(T)]
    din = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(T)]
    dout = [torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(T)]
    sh = [torch.cuda.Stream() for _ in range(T)]
    sd = [torch.cuda.Stream() for _ in range(T)]
    res = {}

    def timed(fn, reps=5):
        best = None
        for _ in range(reps):
            torch.cuda.synchronize()
            time.sleep(0.002)
            a = ev()
            a.record(torch.cuda.current_stream())
            ends = fn(a)
            torch.cuda.synchronize()
            dt = max(a.elapsed_time(e) for e in ends) * 1e3
            best = dt if best is None else min(best, dt)
        return round(best, 1)

    def single(d2h):
        def f(a):
            s = sd[0] if d2h else sh[0]
            s.wait_event(a)
            with torch.cuda.stream(s):
                (hout[0].copy_(dout[0], non_blocking=True) if d2h else din[0].copy_(hin[0], non_blocking=True))
                e = ev()
                e.record(s)
            return [e]
        return f
    res["single_h2d_us"] = timed(single(False))
    res["single_d2h_us"] = timed(single(True))

    def pair(a):
        ends = []
        for s, d2h in ((sh[0], False), (sd[0], True)):
            s.wait_event(a)
            with torch.cuda.stream(s):
                (hout[0].copy_(dout[0], non_blocking=True) if d2h else din[0].copy_(hin[0], non_blocking=True))
                e = ev()
                e.record(s)
                ends.append(e)
        return ends
    res["pair_bidir_us"] = timed(pair)

    def prequeued(a):
        ends = []
        for s, d2h in ((sh[0], False), (sd[0], True)):
            s.wait_event(a)
            with torch.cuda.stream(s):
                for _ in range(16):
                    (hout[0].copy_(dout[0], non_blocking=True) if d2h else din[0].copy_(hin[0], non_blocking=True))
                e = ev()
                e.record(s)
                ends.append(e)
        return ends
    res["prequeued_bidir_16x2_us"] = timed(prequeued)
    res["prequeued_bidir_us_per_copy"] = round(res["prequeued_bidir_16x2_us"] / 16, 1)

    def chains(a, jobs=8, stagger=True):
        ends = []
        for t in range(T):
            sh[t].wait_event(a)
        prev = [None] * T
        for j in range(jobs):
            for t in range(T):
                with torch.cuda.stream(sh[t]):
                    if prev[t] is not None:
                        sh[t].wait_event(prev[t])
                    din[t].copy_(hin[t], non_blocking=True)
                    h = ev()
                    h.record(sh[t])
                sd[t].wait_event(h)
                with torch.cuda.stream(sd[t]):
                    hout[t].copy_(dout[t], non_blocking=True)
                    d = ev()
                    d.record(sd[t])
                prev[t] = d
        return prev
    res["chains2_8jobs_us"] = timed(chains)
    res["chains2_us_per_job_step"] = round(res["chains2_8jobs_us"] / 8, 1)
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
