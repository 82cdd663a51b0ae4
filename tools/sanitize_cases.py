"""Small cases for compute-sanitizer (memcheck / racecheck / synccheck), SURVEY §5.

    compute-sanitizer --tool memcheck python tools/sanitize_cases.py gemm_splitk
    ... attn_decode | attn_prefill | add_ln | engine_t1 | engine_tp2_oneshot | engine_tp2_fused

Each case runs the kernels on tiny shapes through the C ABI and checks the result
against torch so that a sanitizer run also shows the case computed something."""
import os
import sys
import threading

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ppopp_duwjchcl24_b200 import liger as L  # noqa: E402


def ws(nbytes):
    return torch.zeros(max(int(nbytes), 16384) // 4 + 16, dtype=torch.int32, device="cuda")


def gemm_splitk():
    torch.manual_seed(0)
    for M, N, K in ((4, 640, 4096), (8, 384, 2048), (70, 256, 1024)):
        x = (torch.randn(M, K, device="cuda") * 0.5).bfloat16()
        w = (torch.randn(N, K, device="cuda") / K ** 0.5).bfloat16()
        b = (torch.randn(N, device="cuda") * 0.1).bfloat16()
        out = torch.zeros(M, N, device="cuda", dtype=torch.bfloat16)
        L.gemm(x, w, out, bias=b, act="relu", workspace=ws(L.gemm_workspace_bytes(M, N, K)))
        torch.cuda.synchronize()
        ref = torch.relu(x.float() @ w.float().T + b.float())
        err = ((out.float() - ref).abs().max() / ref.abs().max()).item()
        print(f"gemm {M}x{N}x{K} plan {L.gemm_plan(M, N, K)} rel {err:.2e}")
        assert err < 2e-2


def attn_decode():
    torch.manual_seed(1)
    for b, heads, d, pos in ((2, 3, 128, 70), (3, 2, 64, 200), (1, 4, 128, 5)):
        maxp = (pos + 1 + 15) // 16 + 1
        pool = (torch.randn(b * maxp, 2, heads, 16, d, device="cuda") * 0.5).bfloat16()
        pt = torch.arange(b * maxp, dtype=torch.int32, device="cuda").reshape(b, maxp)
        qkv = (torch.randn(b, 3 * heads * d, device="cuda") * 0.5).bfloat16()
        o = torch.zeros(b, heads * d, device="cuda", dtype=torch.bfloat16)
        L.attn_decode(qkv, o, pool, pt, b=b, pos=pos, heads=heads, d=d,
                      workspace=ws(L.attn_decode_workspace_bytes(b, heads, d, pos + 1)))
        torch.cuda.synchronize()
        k = pool[:, 0].reshape(b, maxp, heads, 16, d).permute(0, 2, 1, 3, 4).reshape(b, heads, maxp * 16, d)[:, :, :pos + 1]
        v = pool[:, 1].reshape(b, maxp, heads, 16, d).permute(0, 2, 1, 3, 4).reshape(b, heads, maxp * 16, d)[:, :, :pos + 1]
        q = qkv[:, :heads * d].reshape(b, heads, 1, d).float()
        p = torch.softmax(q @ k.float().transpose(-1, -2), -1)
        ref = (p @ v.float()).reshape(b, heads * d)
        err = ((o.float() - ref).abs().max() / ref.abs().max()).item()
        print(f"attn_decode b={b} heads={heads} d={d} pos={pos} rel {err:.2e}")
        assert err < 2e-2


def attn_prefill():
    torch.manual_seed(2)
    b, s, heads, d = 2, 70, 2, 64
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
    print(f"attn_prefill rel {err:.2e}")
    assert err < 2e-2


def add_ln():
    torch.manual_seed(3)
    R, h = 5, 1024
    x = torch.randn(R, h, device="cuda").bfloat16()
    a = torch.randn(R, h, device="cuda").bfloat16()
    g = torch.rand(h, device="cuda").bfloat16()
    be = torch.randn(h, device="cuda").bfloat16()
    y = torch.empty_like(x)
    L.add_layernorm(x, g, be, y, add=a)
    torch.cuda.synchronize()
    r = (x.float() + a.float()).bfloat16().float()
    ref = torch.nn.functional.layer_norm(r, (h,), g.float(), be.float(), 1e-5)
    err = ((y.float() - ref).abs().max() / ref.abs().max()).item()
    print(f"add_ln rel {err:.2e}")
    assert err < 2e-2


def _engine(world, env):
    os.environ.update(env)
    from liger_inputs import get_config, make_trace
    from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
    from liger_inputs.configs import ModelConfig
    cfg = get_config("tiny")
    trace = make_trace(2, float("inf"), seed=1, batch_sizes=(1, 2), prompt_range=(8, 24), n_decode=3,
                       vocab=cfg.vocab)
    uid = LigerEngine.loopback_id() if world > 1 else None
    toks = [None] * world
    err = []

    def run(r):
        try:
            torch.cuda.set_device(0)
            e = LigerEngine(cfg, world=world, rank=r, nccl_uid=uid, mode="interleaved", max_batch=2, max_seq=32,
                            max_new=4, seed=0)
            ids = [e.submit(t["tokens"], t["batch"], t["seq_len"], t["n_decode"], 0.0) for t in trace]
            e.drain()
            toks[r] = [e.poll(i, want_tokens=True)[1].tolist() for i in ids]
            e.close()
        except Exception as ex:
            err.append(repr(ex))
    ths = [threading.Thread(target=run, args=(r,), daemon=True) for r in range(world)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    assert not err, err
    assert all(t == toks[0] for t in toks)
    print(f"engine world={world} {env}: tokens {toks[0]}")


def _peer_ar_phased():
    """One-shot and fused GEMM + all-reduce kernels at t = 2, phase by phase on one GPU
    (every rank's stage / publish launch completes before any rank's wait / sum launch)."""
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
    import test_gpu_peer_ar as T
    from paper_conf_ppopp_duwjchcl24_b200 import liger
    T.test_oneshot_allreduce_phased_vs_oracle(liger, 2)
    T.test_fused_gemm_allreduce_phased_vs_oracle(liger, 2)
    print("peer_ar phased ok")


CASES = {
    "gemm_splitk": gemm_splitk, "attn_decode": attn_decode, "attn_prefill": attn_prefill, "add_ln": add_ln,
    "engine_t1": lambda: _engine(1, {}),
    "engine_tp2_loopback": lambda: _engine(2, {}),
    "peer_ar_phased": lambda: _peer_ar_phased(),
}

if __name__ == "__main__":
    for name in sys.argv[1:] or list(CASES):
        CASES[name]()
    print("ok")
