"""Dev: one prefill-attention launch (OPT-13B heads / d) for ncu.  python tools/ncu_attn_prefill.py b s"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
b, s = (int(a) for a in (sys.argv[1:3] if len(sys.argv) > 2 else (8, 128)))
heads, d = 40, 128
maxp = (s + 15) // 16 + 1
pool = torch.zeros(b * maxp, 2, heads, 16, d, device="cuda", dtype=torch.bfloat16)
pt = torch.arange(b * maxp, dtype=torch.int32, device="cuda").reshape(b, maxp)
qkv = (torch.randn(b * s, 3 * heads * d, device="cuda") * 0.5).bfloat16()
o = torch.empty(b * s, heads * d, device="cuda", dtype=torch.bfloat16)
for _ in range(3):
    L.attn_prefill(qkv, o, pool, pt, b=b, s=s, heads=heads, d=d)
torch.cuda.synchronize()
