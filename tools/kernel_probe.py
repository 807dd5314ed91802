"""Launch each tenant kernel stand-alone at its ncu size (for ncu captures).

    ncu --set full --clock-control none --import-source on -k regex:oneshot -c 6 \
        -o gpurun_out/prof python tools/kernel_probe.py

Order of launches: VSCALE n=2^28 (x2), XFER n=2^28 (x2), GEMM 18944x256x256 R=64 (x2);
`xfer_item`: XFER n=2^24 on 72 then 144 CTAs (x2 each), the C2 work item on one P=2 partition;
`hist` (2^30 bytes), `scan`, `sort` (2^28 u32): the NEXT-2 bodies; `gemm_small`: the C2 job's GEMM
(256^3, R = 64) on 2 CTAs, SURVEY 8(d)'s tensor-pipe check.
The persistent dispatcher runs exactly these device bodies on its SM partitions.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402


def main():
    which = sys.argv[1:] or ["vscale", "xfer", "gemm"]
    st = torch.cuda.current_stream().cuda_stream
    n = 1 << 28
    if "vscale" in which or "xfer" in which:
        x = torch.empty(n, dtype=torch.float32, device="cuda").uniform_(-1, 1)
        y = torch.empty_like(x)
        for cls, name in ((S.VSCALE, "vscale"), (S.XFER, "xfer")):
            if name in which:
                for _ in range(2):
                    S.kernel_launch(0, S.make_desc(cls, n=n, alpha=1.001, seed=7), [x.data_ptr()], [y.data_ptr()],
                                    stream=st)
        torch.cuda.synchronize()
        del x, y
    if "xfer_item" in which:
        # the C2 work item as the dispatcher runs it: XFER 2^24 u32 on one 72-SM KL
        # partition (148 SMs - 4 copy-partition CTAs, P = 2), and on 144 SMs (an idle
        # sibling slot lending its CTAs); 4 rotating buffer pairs (512 MiB > L2)
        n24 = 1 << 24
        xs = [torch.randint(0, 1 << 30, (n24,), dtype=torch.int32, device="cuda") for _ in range(4)]
        ys = [torch.empty_like(x) for x in xs]
        for ctas in (72, 144):
            for i in range(2):
                S.kernel_launch(0, S.make_desc(S.XFER, n=n24, seed=7), [xs[i].data_ptr()], [ys[i].data_ptr()],
                                ctas=ctas, stream=st)
        torch.cuda.synchronize()
        del xs, ys
    if "gemm" in which:
        m, nn, k, reps = 128 * 148, 256, 256, 64
        a = torch.randint(-2, 3, (m, k), device="cuda").to(torch.bfloat16)
        b = torch.randint(-2, 3, (k, nn), device="cuda").to(torch.bfloat16)
        c = torch.empty((m, nn), dtype=torch.float32, device="cuda")
        for _ in range(2):
            S.kernel_launch(0, S.make_desc(S.GEMM, m=m, n=nn, k=k, reps=reps), [a.data_ptr(), b.data_ptr()],
                            [c.data_ptr()], stream=st)
        torch.cuda.synchronize()
        assert torch.equal(c, a.float() @ b.float())
    if "gemm_small" in which:
        # SURVEY 8(d)'s kernel check: the C2 job's GEMM (256^3, R = 64) on 2 CTAs, one
        # 128 x 256 tile each with all 64 repetitions (tensor-pipe activity on its SMs)
        m, nn, k, reps = 256, 256, 256, 64
        a = torch.randint(-2, 3, (m, k), device="cuda").to(torch.bfloat16)
        b = torch.randint(-2, 3, (k, nn), device="cuda").to(torch.bfloat16)
        c = torch.empty((m, nn), dtype=torch.float32, device="cuda")
        for _ in range(2):
            S.kernel_launch(0, S.make_desc(S.GEMM, m=m, n=nn, k=k, reps=reps), [a.data_ptr(), b.data_ptr()],
                            [c.data_ptr()], ctas=2, stream=st)
        torch.cuda.synchronize()
        assert torch.equal(c, a.float() @ b.float())
    if "hist" in which:
        nb = 1 << 30
        xb = torch.randint(0, 256, (nb,), dtype=torch.uint8, device="cuda")
        hb = torch.zeros(256, dtype=torch.int32, device="cuda")
        for _ in range(2):
            S.kernel_launch(0, S.make_desc(S.HIST, n=nb), [xb.data_ptr()], [hb.data_ptr()], stream=st)
        torch.cuda.synchronize()
        del xb, hb
    for name, cls in (("scan", S.SCAN), ("sort", S.SORT)):
        if name in which:
            n28 = 1 << 28
            xs = torch.randint(0, 1 << 20, (n28,), dtype=torch.int32, device="cuda")
            ys = torch.empty_like(xs)
            for _ in range(2):
                S.kernel_launch(0, S.make_desc(cls, n=n28), [xs.data_ptr()], [ys.data_ptr()], stream=st)
            torch.cuda.synchronize()
            del xs, ys
    print("probe done")


if __name__ == "__main__":
    main()
