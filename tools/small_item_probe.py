"""Stream bodies on small items: VSCALE/XFER at n = 2^20 / 2^22 (C1/C3's 4 MiB VSCALE
jobs) on 18 / 36 / 72 CTAs (a KL slot of C3 / C1 / C2), stand-alone launches timed
with CUDA events (launch overhead included, the same for every build).

    python tools/small_item_probe.py [label]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_sc_senguptagsp14_b200 import strings as S  # noqa: E402


def main():
    label = sys.argv[1] if len(sys.argv) > 1 else ""
    st = torch.cuda.current_stream()
    for n in (1 << 20, 1 << 22):
        x = torch.empty(n, dtype=torch.float32, device="cuda").uniform_(-1, 1)
        y = torch.empty_like(x)
        for ctas in (18, 36, 72):
            for cls, name in ((S.VSCALE, "VSCALE"), (S.XFER, "XFER")):
                d = S.make_desc(cls, n=n, alpha=1.001, seed=3)
                for _ in range(3):
                    S.kernel_launch(0, d, [x.data_ptr()], [y.data_ptr()], ctas=ctas, stream=st.cuda_stream)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                reps = 50
                e0.record(st)
                for _ in range(reps):
                    S.kernel_launch(0, d, [x.data_ptr()], [y.data_ptr()], ctas=ctas, stream=st.cuda_stream)
                e1.record(st)
                torch.cuda.synchronize()
                us = e0.elapsed_time(e1) * 1e3 / reps
                print(json.dumps({"build": label, "kernel": name, "n": n, "ctas": ctas, "us": round(us, 2),
                                  "GBps": round(8 * n / us / 1e3, 1)}), flush=True)


if __name__ == "__main__":
    main()
