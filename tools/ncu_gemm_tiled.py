"""ncu target: tiled-layout GEMM through liger_op_gemm_tiled (as the engine launches it)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
M, N, K = (int(a) for a in sys.argv[1:4])
x = torch.randn(M, K, device="cuda").bfloat16()
w = (torch.randn(N, K, device="cuda") / K ** 0.5).bfloat16()
wt = torch.empty(L.tiled_numel(N, K), dtype=torch.bfloat16, device="cuda")
L.tile_weight(w, wt)
out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
ws = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 16, dtype=torch.int32, device="cuda")
for _ in range(4):
    L.gemm_tiled(x, wt, out, N=N, workspace=ws)
torch.cuda.synchronize()
