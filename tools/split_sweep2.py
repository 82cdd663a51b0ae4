"""Dev: decode GEMM time (PDL chain of 20 launches over rotating weights) vs forced
split count, per shape: python tools/split_sweep2.py M N K S1,S2,..."""
import sys, os, subprocess, json
if len(sys.argv) > 1 and sys.argv[1] == "child":
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    from paper_conf_ppopp_duwjchcl24_b200 import liger as L
    M, N, K = (int(a) for a in sys.argv[2:5])
    copies = max(2, int(1500e6 // (N * K * 2)))
    ws_ = [torch.empty(L.tiled_numel(N, K), dtype=torch.bfloat16, device="cuda").normal_(0, 0.02) for _ in range(copies)]
    x = torch.randn(M, K, device="cuda").bfloat16()
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    wsp = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 16, dtype=torch.int32, device="cuda")
    g = lambda i: L.gemm_tiled(x, ws_[i % copies], out, N=N, workspace=wsp)
    for i in range(4): g(i)
    torch.cuda.synchronize()
    best = 1e9
    for rep in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for i in range(30): g(i)
        b.record(); torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) / 30 * 1e-3)
    print(json.dumps({"M": M, "N": N, "K": K, "splits": L.gemm_plan(M, N, K)["splits"], "us": round(best * 1e6, 2),
                      "GBs": round(N * K * 2 / best / 1e9)}), flush=True)
else:
    M, N, K = (int(a) for a in sys.argv[1:4])
    for S in [int(s) for s in sys.argv[4].split(",")]:
        env = dict(os.environ)
        if S > 0:
            env["LIGER_GEMM_FORCE_SPLITS"] = str(S)
        r = subprocess.run([sys.executable, __file__, "child", str(M), str(N), str(K)], env=env, capture_output=True, text=True)
        print(r.stdout.strip() or r.stderr[-300:], flush=True)
