"""Dev: fused residual add + LayerNorm (prefill rows, OPT-13B h = 5120) -- CUDA events,
buffers rotated over copies larger than L2.   python tools/kbench_ln.py"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import json, torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
HBM = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"]
h = 5120
g = torch.randn(h, device="cuda").bfloat16()
be = torch.randn(h, device="cuda").bfloat16()
bias = torch.randn(h, device="cuda").bfloat16()
for rows in (512, 1024, 2048, 4096):
    copies = max(2, int(400e6 // (rows * h * 2 * 4)))
    xs = [torch.randn(rows, h, device="cuda").bfloat16() for _ in range(copies)]
    ad = [torch.randn(rows, h, device="cuda").bfloat16() for _ in range(copies)]
    ys = [torch.empty(rows, h, device="cuda", dtype=torch.bfloat16) for _ in range(copies)]
    fn = lambda i: L.add_layernorm(xs[i % copies], g, be, ys[i % copies], add=ad[i % copies], add_bias=bias,
                                   x_out=xs[i % copies])
    for i in range(3):
        fn(i)
    torch.cuda.synchronize()
    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 30
    a.record()
    for i in range(n):
        fn(i)
    e.record(); torch.cuda.synchronize()
    t = a.elapsed_time(e) / n * 1e-3
    by = rows * h * 2 * 4
    print(f"add_ln rows={rows:5d}: {t*1e6:7.1f} us {by/t/1e9:7.0f} GB/s "
          f"({by/t/1e9/HBM*100:4.1f}%)", flush=True)
