import sys, os, torch
sys.path.insert(0, "/root/repo")
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
torch.manual_seed(0)
cases = [tuple(int(x) for x in a.split(",")) for a in sys.argv[1:]]
for (b, s, heads, d) in cases:
    maxp = (s + 15) // 16 + 1
    pool = torch.zeros(b * maxp, 2, heads, 16, d, device="cuda", dtype=torch.bfloat16)
    pt = torch.arange(b * maxp, dtype=torch.int32, device="cuda").reshape(b, maxp)
    qkv = (torch.randn(b * s, 3 * heads * d, device="cuda") * 0.5).bfloat16()
    o = torch.zeros(b * s, heads * d, device="cuda", dtype=torch.bfloat16)
    L.attn_prefill(qkv, o, pool, pt, b=b, s=s, heads=heads, d=d)
    torch.cuda.synchronize()
    q, k, v = qkv.float().reshape(b, s, 3, heads, d).permute(2, 0, 3, 1, 4)
    ref = torch.nn.functional.scaled_dot_product_attention(q, k, v, is_causal=True, scale=1.0)
    ref = ref.permute(0, 2, 1, 3).reshape(b * s, heads * d)
    err = ((o.float() - ref).abs().max() / ref.abs().max()).item()
    print(f"b={b} s={s} heads={heads} d={d}: rel {err:.3e}", flush=True)
