"""Target for `ncu --set full`: the decode (and prefill) GEMM through liger_op_gemm."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
M, N, K = (int(a) for a in sys.argv[1:4])
x = torch.randn(M, K, device="cuda").bfloat16(); w = (torch.randn(N, K, device="cuda") / K ** 0.5).bfloat16()
out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
ws = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 16, dtype=torch.int32, device="cuda")
for _ in range(5):
    L.gemm(x, w, out, workspace=ws)
torch.cuda.synchronize()
