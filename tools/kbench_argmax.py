"""Dev: LM-head argmax over the OPT vocabulary (50272 fp32 logits per row), CUDA events."""
import sys, os
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
for rows in (2, 8, 32):
    d = [torch.randn(rows, 50272, device="cuda") for _ in range(64)]
    mx = torch.empty(rows, device="cuda"); ix = torch.empty(rows, dtype=torch.int32, device="cuda")
    for i in range(3): L.argmax(d[i], mx, ix)
    torch.cuda.synchronize()
    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for i in range(64): L.argmax(d[i], mx, ix)
    e.record(); torch.cuda.synchronize()
    print(f"argmax rows={rows} n=50272: {a.elapsed_time(e)/64*1e3:.1f} us")
