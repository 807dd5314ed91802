"""Time the SCAN body stand-alone at 2^28 u32 (CUDA events, 10 launches) and check it."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_senguptagsp14_b200 import strings as S
n = 1 << 28
x = torch.randint(0, 1 << 20, (n,), dtype=torch.int32, device="cuda")
y = torch.empty_like(x)
st = torch.cuda.current_stream()
d = S.make_desc(S.SCAN, n=n)
for ctas in (0, 74):
    S.kernel_launch(0, d, [x.data_ptr()], [y.data_ptr()], ctas=ctas, stream=st.cuda_stream)
    torch.cuda.synchronize()
    ref = torch.cumsum(x.to(torch.int64), 0).to(torch.int64) & 0xFFFFFFFF
    ok = torch.equal((y.to(torch.int64) & 0xFFFFFFFF), ref)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(10):
        S.kernel_launch(0, d, [x.data_ptr()], [y.data_ptr()], ctas=ctas, stream=st.cuda_stream)
    e1.record(st)
    torch.cuda.synchronize()
    t = e0.elapsed_time(e1) / 10 / 1e3
    print(f"ctas {ctas or 148}: {t*1e3:.3f} ms, {8*n/t/1e9:.0f} GB/s, exact {ok}")
