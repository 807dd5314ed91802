"""SCAN body stand-alone: exactness over ragged sizes and CTA counts, then the
2^28 u32 timing (CUDA events, 10 launches) on 148 and 74 CTAs."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_senguptagsp14_b200 import strings as S
st = torch.cuda.current_stream()


def run(n, ctas, x=None):
    x = torch.randint(0, 1 << 20, (max(n, 1),), dtype=torch.int32, device="cuda")[:n] if x is None else x
    y = torch.empty_like(x)
    S.kernel_launch(0, S.make_desc(S.SCAN, n=n), [x.data_ptr()], [y.data_ptr()], ctas=ctas, stream=st.cuda_stream)
    torch.cuda.synchronize()
    ref = torch.cumsum(x.to(torch.int64), 0) & 0xFFFFFFFF
    return torch.equal(y.to(torch.int64) & 0xFFFFFFFF, ref), x, y


quick = "--quick" in sys.argv
bad = 0
for n in () if quick else (0, 1, 100, 24575, 24576, 24577, 3 * 24576 + 5, (1 << 20) + 7, 1 << 24):
    for ctas in (1, 3, 37, 148):
        if n == 0:
            continue
        ok, _, _ = run(n, ctas)
        bad += not ok
        if not ok:
            print("MISMATCH n", n, "ctas", ctas, flush=True)
print("sweep mismatches:", bad, flush=True)
n = 1 << 28
x = torch.randint(0, 1 << 20, (n,), dtype=torch.int32, device="cuda")
y = torch.empty_like(x)
d = S.make_desc(S.SCAN, n=n)
for ctas in ((0,) if quick else (0, 74)):
    ok, _, _ = run(n, ctas, x)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(1 if "--once" in sys.argv else 10):
        S.kernel_launch(0, d, [x.data_ptr()], [y.data_ptr()], ctas=ctas, stream=st.cuda_stream)
    e1.record(st)
    torch.cuda.synchronize()
    t = e0.elapsed_time(e1) / 10 / 1e3
    print(f"ctas {ctas or 148}: {t*1e3:.3f} ms, {8*n/t/1e9:.0f} GB/s, exact {ok}", flush=True)
