"""Dev: prefill projection GEMMs (OPT-13B TP=1 shapes) over the bench's prompt-token
range, CUDA events, weights rotated over copies (L2 cold).  Prints TF/s and the plan.
    [LIGER_GEMM_PLAN_V1=1] python tools/kbench_prefill.py"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import json, torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
TC = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["bf16_tflops"]
h, f = 5120, 20480
shapes = ((3 * h, h, "qkv"), (h, h, "out"), (f, h, "fc1"), (h, f, "fc2"))
W = {}
for (N, K, name) in shapes:
    copies = max(2, int(400e6 // (N * K * 2)))
    W[name] = []
    for _ in range(copies):
        w = (torch.randn(N, K, device="cuda") / K ** 0.5).bfloat16()
        wt = torch.empty(L.tiled_numel(N, K), dtype=torch.bfloat16, device="cuda")
        L.tile_weight(w, wt); W[name].append(wt); del w
tot = {}
for M in [int(a) for a in (sys.argv[1:] or [256, 384, 512, 768, 1024, 1536, 2048, 3072, 4096])]:
    for (N, K, name) in shapes:
        x = torch.randn(M, K, device="cuda").bfloat16()
        out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
        wsp = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 16, dtype=torch.int32, device="cuda")
        ws_ = W[name]
        for i in range(3): L.gemm_tiled(x, ws_[i % len(ws_)], out, N=N, workspace=wsp)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        n = 20
        a.record()
        for i in range(n): L.gemm_tiled(x, ws_[i % len(ws_)], out, N=N, workspace=wsp)
        b.record(); torch.cuda.synchronize()
        t = a.elapsed_time(b) / n * 1e-3
        tf = 2 * M * N * K / t / 1e12
        tot[M] = tot.get(M, 0) + t
        print(f"M={M:5d} {name:4s} {t*1e6:8.1f} us {tf:7.1f} TF/s ({tf/TC*100:5.1f}%) plan {L.gemm_plan(M, N, K)}", flush=True)
print("per-layer GEMM time (us):", {m: round(v * 1e6, 1) for m, v in tot.items()})
