"""Dev: decode projection GEMMs (OPT-13B TP=1, M = b tokens) isolated, CUDA events,
weights rotated over copies (L2 cold).  python tools/kbench_decode.py [M ...]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import json, torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
HBM = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"]
h, f = 5120, 20480
shapes = ((3 * h, h, "qkv"), (h, h, "out"), (f, h, "fc1"), (h, f, "fc2"))
for M in [int(a) for a in (sys.argv[1:] or [8])]:
    tot = 0.0
    for (N, K, name) in shapes:
        copies = max(2, int(600e6 // (N * K * 2)))
        ws_ = []
        for _ in range(copies):
            wt = torch.empty(L.tiled_numel(N, K), dtype=torch.bfloat16, device="cuda").normal_(0, 0.02)
            ws_.append(wt)
        x = torch.randn(M, K, device="cuda").bfloat16()
        out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
        wsp = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 16, dtype=torch.int32, device="cuda")
        for i in range(3): L.gemm_tiled(x, ws_[i % copies], out, N=N, workspace=wsp)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        n = 30
        a.record()
        for i in range(n): L.gemm_tiled(x, ws_[i % copies], out, N=N, workspace=wsp)
        b.record(); torch.cuda.synchronize()
        t = a.elapsed_time(b) / n * 1e-3
        tot += t
        by = (N * K + M * K + M * N) * 2
        print(f"M={M:3d} {name:4s} {t*1e6:7.1f} us {by/t/1e9:6.0f} GB/s ({by/t/1e9/HBM*100:5.1f}%) plan {L.gemm_plan(M, N, K)}", flush=True)
        del ws_
    print(f"M={M} layer GEMMs {tot*1e6:.1f} us")
