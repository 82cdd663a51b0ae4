"""Dev experiment: decode GEMM time vs forced split count (LIGER_GEMM_FORCE_SPLITS)."""
import sys, os, subprocess, json
if len(sys.argv) > 1 and sys.argv[1] == "child":
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    from paper_conf_ppopp_duwjchcl24_b200 import liger as L
    M, N, K = (int(a) for a in sys.argv[2:5])
    copies = max(1, int(600e6 // (N * K * 2)))
    ws_ = []
    for _ in range(copies):
        w = (torch.randn(N, K, device="cuda") / K ** 0.5).bfloat16()
        wt = torch.empty(L.tiled_numel(N, K), dtype=torch.bfloat16, device="cuda")
        L.tile_weight(w, wt)
        ws_.append(wt)
        del w
    x = torch.randn(M, K, device="cuda").bfloat16()
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    wsp = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 16, dtype=torch.int32, device="cuda")
    g = lambda i: L.gemm_tiled(x, ws_[i % copies], out, N=N, workspace=wsp)
    for i in range(3): g(i)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for i in range(20): g(i)
    b.record(); torch.cuda.synchronize()
    t = a.elapsed_time(b) / 20 * 1e-3
    print(json.dumps({"M": M, "N": N, "K": K, "plan": L.gemm_plan(M, N, K), "us": t * 1e6, "GBs": N * K * 2 / t / 1e9}))
else:
    for (M, N, K) in ((8, 20480, 5120), (8, 15360, 5120), (8, 5120, 5120), (8, 5120, 20480), (256, 5120, 5120), (1024, 5120, 20480)):
        for S in (1, 2, 3, 4, 5, 8, 10, 16):
            env = dict(os.environ, LIGER_GEMM_FORCE_SPLITS=str(S))
            r = subprocess.run([sys.executable, __file__, "child", str(M), str(N), str(K)], env=env, capture_output=True, text=True)
            print(r.stdout.strip() or r.stderr[-300:], flush=True)
