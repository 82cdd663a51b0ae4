"""ncu target: the latency-bound decode kernels at OPT-13B TP=1 bench shapes (b = 8):
add + LN, out-proj GEMM with its split-K fixup, decode attention (ctx 300), LM head."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
b, h, heads, d, ctx, V = 8, 5120, 40, 128, 300, 50272
maxp = (ctx + 16) // 16 + 1
pool = torch.randn(b * maxp, 2, heads, 16, d, device="cuda").bfloat16()
pt = torch.arange(b * maxp, dtype=torch.int32, device="cuda").reshape(b, maxp)
qkv = torch.randn(b, 3 * heads * d, device="cuda").bfloat16()
o = torch.empty(b, heads * d, device="cuda", dtype=torch.bfloat16)
aws = torch.zeros(L.attn_decode_workspace_bytes(b, heads, d, ctx + 1) // 4 + 16, dtype=torch.int32, device="cuda")
x = torch.randn(b, h, device="cuda").bfloat16(); a = torch.randn(b, h, device="cuda").bfloat16()
g = torch.randn(h, device="cuda").bfloat16(); y = torch.empty_like(x)
wo = torch.empty(L.tiled_numel(h, h), dtype=torch.bfloat16, device="cuda")
L.tile_weight((torch.randn(h, h, device="cuda") * 0.01).bfloat16(), wo)
part = torch.empty(b, h, device="cuda", dtype=torch.bfloat16)
gws = torch.zeros(L.gemm_workspace_bytes(b, h, h) // 4 + 16, dtype=torch.int32, device="cuda")
emb = (torch.randn(V, h, device="cuda") * 0.02).bfloat16()
logits = torch.empty(b, V, device="cuda", dtype=torch.float32)
hws = torch.zeros(max(L.gemm_workspace_bytes(b, V, h), 16384) // 4 + 16, dtype=torch.int32, device="cuda")
for _ in range(3):
    L.add_layernorm(x, g, g, y, add=a, add_bias=g, x_out=x)
    L.gemm_tiled(o, wo, part, N=h, workspace=gws)
    L.attn_decode(qkv, o, pool, pt, b=b, pos=ctx, heads=heads, d=d, workspace=aws)
    L.gemm(y, emb, logits, workspace=hws)
torch.cuda.synchronize()
print("done")
