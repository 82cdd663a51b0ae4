"""Dev: prefill attention (OPT-13B: 40 heads, d = 128) at the bench's prompt shapes,
CUDA events.  Causal flops = 2 * 2 * b * heads * d * s (s + 1) / 2.
    [LIGER_ATTN_PREFILL_MMA_SYNC=1] python tools/kbench_attn_prefill.py"""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
TC = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["bf16_tflops"]
heads, d = 40, 128
for (b, s) in ((2, 128), (2, 512), (4, 256), (8, 128), (8, 384), (8, 512)):
    maxp = (s + 15) // 16 + 1
    pool = torch.zeros(b * maxp, 2, heads, 16, d, device="cuda", dtype=torch.bfloat16)
    pt = torch.arange(b * maxp, dtype=torch.int32, device="cuda").reshape(b, maxp)
    qkv = (torch.randn(b * s, 3 * heads * d, device="cuda") * 0.5).bfloat16()
    o = torch.empty(b * s, heads * d, device="cuda", dtype=torch.bfloat16)
    f = lambda: L.attn_prefill(qkv, o, pool, pt, b=b, s=s, heads=heads, d=d)
    for _ in range(3): f()
    torch.cuda.synchronize()
    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 20
    a.record()
    for _ in range(n): f()
    e.record(); torch.cuda.synchronize()
    t = a.elapsed_time(e) / n * 1e-3
    fl = 2 * 2 * b * heads * d * s * (s + 1) / 2
    print(f"attn_prefill b={b} s={s}: {t*1e6:7.1f} us {fl/t/1e12:6.1f} TF/s ({fl/t/1e12/TC*100:4.1f}% of bf16 peak)", flush=True)
