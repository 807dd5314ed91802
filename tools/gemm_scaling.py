"""GEMM time vs repetitions R on 148 CTAs (one 128x256 tile each): T(R) = a + b*R."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sc_senguptagsp14_b200 import strings as S

m, n, k = 128 * 148, 256, 256
a = torch.randint(-2, 3, (m, k), device="cuda").to(torch.bfloat16)
b = torch.randint(-2, 3, (k, n), device="cuda").to(torch.bfloat16)
c = torch.empty((m, n), dtype=torch.float32, device="cuda")
st = torch.cuda.current_stream()
out = {}
for R in (1, 2, 4, 16, 64, 256):
    d = S.make_desc(S.GEMM, m=m, n=n, k=k, reps=R)
    for _ in range(3):
        S.kernel_launch(0, d, [a.data_ptr(), b.data_ptr()], [c.data_ptr()], stream=st.cuda_stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(20):
        S.kernel_launch(0, d, [a.data_ptr(), b.data_ptr()], [c.data_ptr()], stream=st.cuda_stream)
    e1.record(st)
    torch.cuda.synchronize()
    t = e0.elapsed_time(e1) / 20 * 1e3
    out[R] = round(t, 2)
print(json.dumps({"us_by_R": out, "per_rep_us_64_to_256": round((out[256] - out[64]) / 192, 4),
                  "ideal_per_rep_us_at_1965MHz": round(2048 / 1965, 4)}))
