"""Dev: decode attention (OPT-13B TP=1: 40 heads of 128) at the bench's batch sizes and
contexts; CUDA events, KV pools rotated over copies larger than L2.
    [LIGER_ATTN_V1=1] python tools/kbench_attn.py"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import json, torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
HBM = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"]
heads, d = 40, 128
for (b, ctx) in ((2, 160), (2, 300), (4, 300), (8, 300), (8, 540), (32, 48)):
    maxp = (ctx + 16) // 16 + 1
    copies = max(2, int(300e6 // (b * maxp * 2 * heads * 16 * d * 2)))
    pools = [torch.randn(b * maxp, 2, heads, 16, d, device="cuda").bfloat16() for _ in range(copies)]
    pt = torch.randperm(b * maxp, device="cuda").to(torch.int32).reshape(b, maxp)
    qkv = torch.randn(b, 3 * heads * d, device="cuda").bfloat16()
    o = torch.empty(b, heads * d, device="cuda", dtype=torch.bfloat16)
    ws = torch.zeros(L.attn_decode_workspace_bytes(b, heads, d, ctx + 1) // 4 + 16, dtype=torch.int32, device="cuda")
    fn = lambda i: L.attn_decode(qkv, o, pools[i % copies], pt, b=b, pos=ctx, heads=heads, d=d, workspace=ws)
    for i in range(3): fn(i)
    torch.cuda.synchronize()
    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 50
    a.record()
    for i in range(n): fn(i)
    e.record(); torch.cuda.synchronize()
    t = a.elapsed_time(e) / n * 1e-3
    by = b * heads * d * 2 * 2 * (ctx + 1)
    print(f"attn_decode b={b:2d} ctx={ctx:4d}: {t*1e6:7.1f} us {by/t/1e9:7.0f} GB/s ({by/t/1e9/HBM*100:4.1f}%)", flush=True)
