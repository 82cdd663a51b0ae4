"""ncu target: decode attention + LN at bench shapes."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
heads, d, b, ctx = 40, 128, 8, 300
maxp = (ctx + 16) // 16 + 1
pool = torch.randn(b * maxp, 2, heads, 16, d, device="cuda").bfloat16()
pt = torch.arange(b * maxp, dtype=torch.int32, device="cuda").reshape(b, maxp)
qkv = torch.randn(b, 3 * heads * d, device="cuda").bfloat16()
o = torch.empty(b, heads * d, device="cuda", dtype=torch.bfloat16)
ws = torch.zeros(L.attn_decode_workspace_bytes(b, heads, d, ctx + 1) // 4 + 16, dtype=torch.int32, device="cuda")
h = 5120
x = torch.randn(8, h, device="cuda").bfloat16(); a = torch.randn(8, h, device="cuda").bfloat16()
g = torch.randn(h, device="cuda").bfloat16(); y = torch.empty_like(x)
for _ in range(3):
    L.attn_decode(qkv, o, pool, pt, b=b, pos=ctx, heads=heads, d=d, workspace=ws)
    L.add_layernorm(x, g, g, y, add=a, add_bias=g, x_out=x)
torch.cuda.synchronize()
