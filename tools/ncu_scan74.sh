python -m paper_conf_sc_senguptagsp14_b200.build >/dev/null 2>&1
cat > /tmp/scan74.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_sc_senguptagsp14_b200 import strings as S
n = 1 << 28
x = torch.randint(0, 1 << 20, (n,), dtype=torch.int32, device="cuda"); y = torch.empty_like(x)
st = torch.cuda.current_stream()
for c in (74, 74):
    S.kernel_launch(0, S.make_desc(S.SCAN, n=n), [x.data_ptr()], [y.data_ptr()], ctas=c, stream=st.cuda_stream)
torch.cuda.synchronize()
PY
timeout 600 ncu --set full --import-source on --clock-control none -k regex:oneshot_kernel --launch-skip 1 -c 1 -o gpurun_out/scan74 python /tmp/scan74.py > gpurun_out/scan74.log 2>&1
tail -3 gpurun_out/scan74.log
