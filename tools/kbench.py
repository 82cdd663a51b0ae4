"""Kernel micro-benchmarks at the bench's OPT-13B TP=1 shapes (dev tool).
CUDA-event timing, warm L2 excluded by rotating over several weight copies."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
dev = "cuda"
HBM, TC = 6538.0, 1656.6

def timeit(fn, n=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e-3

h, f = 5120, 20480
for M in (2, 8, 32, 256, 512, 1024, 4096):
    for (N, K, name) in ((3 * h, h, "qkv"), (h, h, "out"), (f, h, "fc1"), (h, f, "fc2")):
        copies = max(1, int(600e6 // (N * K * 2)))
        ws_ = []
        for _ in range(copies):
            w = (torch.randn(N, K, device=dev) / K ** 0.5).bfloat16()
            wt = torch.empty(L.tiled_numel(N, K), dtype=torch.bfloat16, device=dev)
            L.tile_weight(w, wt)
            ws_.append(wt)
            del w
        x = torch.randn(M, K, device=dev).bfloat16()
        out = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
        wsp = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 16, dtype=torch.int32, device=dev)
        i = [0]
        def fn():
            L.gemm_tiled(x, ws_[i[0] % copies], out, N=N, workspace=wsp); i[0] += 1
        t = timeit(fn)
        by = (N * K + M * K + M * N) * 2
        print(f"gemm {name:4s} M={M:5d} N={N:6d} K={K:6d}: {t*1e6:8.1f} us  {by/t/1e9:7.0f} GB/s ({by/t/1e9/HBM*100:4.1f}%)  {2*M*N*K/t/1e12:7.1f} TF/s ({2*M*N*K/t/1e12/TC*100:4.1f}%)")
        del ws_
heads, d = 40, 128
for (b, ctx) in ((2, 300), (4, 300), (8, 300), (8, 540)):
    maxp = (ctx + 16) // 16 + 1
    pool = torch.randn(b * maxp, 2, heads, 16, d, device=dev).bfloat16()
    pt = torch.arange(b * maxp, dtype=torch.int32, device=dev).reshape(b, maxp)
    qkv = torch.randn(b, 3 * heads * d, device=dev).bfloat16()
    o = torch.empty(b, heads * d, device=dev, dtype=torch.bfloat16)
    ws = torch.zeros(L.attn_decode_workspace_bytes(b, heads, d, ctx + 1) // 4 + 16, dtype=torch.int32, device=dev)
    t = timeit(lambda: L.attn_decode(qkv, o, pool, pt, b=b, pos=ctx, heads=heads, d=d, workspace=ws))
    by = b * heads * d * 2 * 2 * (ctx + 1)
    print(f"attn_decode b={b} ctx={ctx}: {t*1e6:7.1f} us {by/t/1e9:7.0f} GB/s ({by/t/1e9/HBM*100:4.1f}%)")
for (b, s) in ((4, 256), (8, 512)):
    maxp = (s + 16) // 16 + 1
    pool = torch.zeros(b * maxp, 2, heads, 16, d, device=dev).bfloat16()
    pt = torch.arange(b * maxp, dtype=torch.int32, device=dev).reshape(b, maxp)
    qkv = torch.randn(b * s, 3 * heads * d, device=dev).bfloat16()
    o = torch.empty(b * s, heads * d, device=dev, dtype=torch.bfloat16)
    t = timeit(lambda: L.attn_prefill(qkv, o, pool, pt, b=b, s=s, heads=heads, d=d))
    fl = 2 * b * heads * d * s * s
    print(f"attn_prefill b={b} s={s}: {t*1e6:7.1f} us {fl/t/1e12:6.1f} TF/s")
for R in (2, 8, 512, 4096):
    x = torch.randn(R, h, device=dev).bfloat16(); a = torch.randn(R, h, device=dev).bfloat16()
    g = torch.randn(h, device=dev).bfloat16(); bb = torch.randn(h, device=dev).bfloat16()
    y = torch.empty_like(x)
    t = timeit(lambda: L.add_layernorm(x, g, bb, y, add=a, add_bias=bb, x_out=x))
    by = R * h * 2 * 4
    print(f"add_ln rows={R}: {t*1e6:7.1f} us {by/t/1e9:7.0f} GB/s")
