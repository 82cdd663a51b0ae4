"""Dev: decode GEMM chain (QKV -> out -> FC1 -> FC2) over 40 layers with distinct
tiled weights, as the engine issues them (PDL chain); per-layer device time."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
M = int(sys.argv[1]) if len(sys.argv) > 1 else 8
h, f, Lyr = 5120, 20480, 40
shapes = [(3 * h, h), (h, h), (f, h), (h, f)]
W = [[torch.empty(L.tiled_numel(N, K), dtype=torch.bfloat16, device="cuda").normal_(0, 0.02) for (N, K) in shapes]
     for _ in range(Lyr)]
x = {K: torch.randn(M, K, device="cuda").bfloat16() for K in (h, f)}
outs = {N: torch.empty(M, N, device="cuda", dtype=torch.bfloat16) for (N, _) in shapes}
ws = torch.zeros(max(L.gemm_workspace_bytes(M, N, K) for (N, K) in shapes) // 4 + 16, dtype=torch.int32, device="cuda")
def layer(l):
    for (N, K), w in zip(shapes, W[l]):
        L.gemm_tiled(x[K], w, outs[N], N=N, workspace=ws)
for l in range(Lyr): layer(l)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for r in range(3):
    for l in range(Lyr): layer(l)
b.record(); torch.cuda.synchronize()
t = a.elapsed_time(b) / 3 / Lyr * 1e-3
by = sum(N * K * 2 for N, K in shapes)
print(f"M={M} stages={os.environ.get('LIGER_GEMM_STAGES', 'default')}: {t * 1e6:.1f} us/layer, {by / t / 1e9:.0f} GB/s "
      f"({by / t / 1e9 / 6538 * 100:.1f}% of HBM); plans {[L.gemm_plan(M, N, K)['splits'] for N, K in shapes]}")
