"""Fused decode pass (liger_op_decode_fused, csrc/decode_fused.cu) against the same
layers run op by op through the C ABI (liger_op_add_layernorm, liger_op_gemm_tiled,
liger_op_attn_decode): every output buffer and the KV cache must be bit-identical
(same split plans, MMA K order, reduction orders and LayerNorm tree by design).
The per-op path itself is pinned to the fp64 oracle in test_gpu_parity.py; the
engine test below checks the fused engine's greedy tokens against the oracle."""
import os

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def L():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_duwjchcl24_b200 import liger
    return liger


def _tiled(L, N, K, gen):
    w = (torch.randn(N, K, generator=gen) * K ** -0.5).to(torch.bfloat16).cuda()
    wt = torch.empty(L.tiled_numel(N, K), dtype=torch.bfloat16, device="cuda")
    L.tile_weight(w, wt)
    return wt


def _layer(L, h, heads, d, ffn, gen):
    hl = heads * d
    vec = lambda n, s=0.05: (torch.randn(n, generator=gen) * s).to(torch.bfloat16).cuda()
    gam = lambda n: (1 + torch.randn(n, generator=gen) * 0.1).to(torch.bfloat16).cuda()
    return dict(w_qkv=_tiled(L, 3 * hl, h, gen), w_o=_tiled(L, h, hl, gen), w_1=_tiled(L, ffn, h, gen),
                w_2=_tiled(L, h, ffn, gen), b_qkv=vec(3 * hl), b_o=vec(h), b_1=vec(ffn), b_2=vec(h),
                g1=gam(h), be1=vec(h), g2=gam(h), be2=vec(h))


def _run_case(L, *, n_layers, h, heads, d, ffn, M, pos, act="relu", seed=0):
    gen = torch.Generator().manual_seed(seed)
    hl = heads * d
    layers = [_layer(L, h, heads, d, ffn, gen) for _ in range(n_layers)]
    max_pages = (pos + 1 + 15) // 16 + 1
    n_pages = M * max_pages
    layer_elems = n_pages * 2 * heads * 16 * d
    kv0 = (torch.randn(n_layers * layer_elems, generator=gen) * 0.5).to(torch.bfloat16).cuda()
    page_table = torch.randperm(n_pages, generator=gen).to(torch.int32).reshape(M, max_pages).cuda()
    x0 = (torch.randn(M, h, generator=gen) * 0.5).to(torch.bfloat16).cuda()
    part0 = (torch.randn(M, h, generator=gen) * 0.1).to(torch.bfloat16).cuda()
    ws_bytes = max(L.gemm_workspace_bytes(M, N, K) for N, K in ((3 * hl, h), (h, hl), (ffn, h), (h, ffn)))
    qscale = float(np.float32(1.0) / np.sqrt(np.float32(d)))

    def bufs():
        return dict(x=x0.clone(), y=torch.zeros(M, h, dtype=torch.bfloat16, device="cuda"),
                    qkv=torch.zeros(M, 3 * hl, dtype=torch.bfloat16, device="cuda"),
                    attn=torch.zeros(M, hl, dtype=torch.bfloat16, device="cuda"), part=part0.clone(),
                    hbuf=torch.zeros(M, ffn, dtype=torch.bfloat16, device="cuda"), kv=kv0.clone(),
                    gws=torch.zeros(ws_bytes // 4 + 16, dtype=torch.int32, device="cuda"),
                    aws=torch.zeros(L.attn_decode_workspace_bytes(M, heads, d, pos + 1) // 4 + 16,
                                    dtype=torch.int32, device="cuda"))

    # op by op (the engine's per-kernel decode path)
    B = bufs()
    for l, W in enumerate(layers):
        if l == 0:
            L.add_layernorm(B["x"], W["g1"], W["be1"], B["y"])
        else:
            L.add_layernorm(B["x"], W["g1"], W["be1"], B["y"], add=B["part"], add_bias=layers[l - 1]["b_2"],
                            x_out=B["x"])
        L.gemm_tiled(B["y"], W["w_qkv"], B["qkv"], N=3 * hl, bias=W["b_qkv"], scale_cols=hl, scale=qscale,
                     workspace=B["gws"])
        L.attn_decode(B["qkv"], B["attn"], B["kv"][l * layer_elems:], page_table, b=M, pos=pos, heads=heads, d=d,
                      workspace=B["aws"])
        L.gemm_tiled(B["attn"], W["w_o"], B["part"], N=h, workspace=B["gws"])
        L.add_layernorm(B["x"], W["g2"], W["be2"], B["y"], add=B["part"], add_bias=W["b_o"], x_out=B["x"])
        L.gemm_tiled(B["y"], W["w_1"], B["hbuf"], N=ffn, bias=W["b_1"], act=act, workspace=B["gws"])
        L.gemm_tiled(B["hbuf"], W["w_2"], B["part"], N=h, workspace=B["gws"])
    torch.cuda.synchronize()

    Fz = bufs()
    L.decode_fused(layers, M=M, h=h, heads=heads, d=d, ffn=ffn, act=act, pos=pos, x=Fz["x"], y=Fz["y"],
                   qkv=Fz["qkv"], attn=Fz["attn"], part=Fz["part"], hbuf=Fz["hbuf"], kv=Fz["kv"],
                   kv_layer_elems=layer_elems, page_table=page_table, max_pages=max_pages, gemm_ws=Fz["gws"],
                   attn_ws=Fz["aws"], qscale=qscale)
    torch.cuda.synchronize()
    for k in ("x", "y", "qkv", "attn", "part", "hbuf", "kv"):
        a, b = B[k], Fz[k]
        bad = (a.view(torch.int16) != b.view(torch.int16)).sum().item()
        assert bad == 0, f"{k}: {bad} elements differ (max |diff| {(a.float() - b.float()).abs().max().item()})"
    # counters left zero for the next user
    assert int(Fz["gws"][:4096].abs().sum().item()) == 0
    assert int(Fz["aws"][:4096].abs().sum().item()) == 0
    return Fz


@pytest.mark.parametrize("M,pos", [(1, 0), (2, 5), (8, 70), (8, 300), (24, 33), (32, 129)])
def test_fused_equals_per_op_d128(L, M, pos):
    _run_case(L, n_layers=2, h=1024, heads=8, d=128, ffn=4096, M=M, pos=pos)


def test_fused_equals_per_op_tiny_d64_gelu(L):
    # BASELINE.json configs[0] shapes at t = 1 (h 256, 4 heads of 64, ffn 1024), tanh-GELU
    _run_case(L, n_layers=2, h=256, heads=4, d=64, ffn=1024, M=2, pos=40, act="gelu_tanh")


def test_fused_equals_per_op_opt13b_layer(L):
    # OPT-13B at t = 1 (BASELINE.json configs[1] shapes, one sharded rank of TP=1), the bench's
    # decode shape: real split plans (QKV unsplit, out/FC1/FC2 split-K)
    _run_case(L, n_layers=1, h=5120, heads=40, d=128, ffn=20480, M=8, pos=300)


def test_fused_repeated_launches(L):
    # the cross-CTA phase counter is never reset: consecutive launches use fresh targets
    for i in range(3):
        _run_case(L, n_layers=1, h=512, heads=4, d=128, ffn=2048, M=4, pos=17 + i, seed=i)


def test_engine_fused_tokens_equal_per_op_and_oracle():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from liger_inputs import get_config
    from oracle import model as om
    from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
    cfg = get_config("tiny")
    prompt = np.random.default_rng(5).integers(0, cfg.vocab, size=(3, 20))
    out = {}
    for fused in ("1", "0"):
        os.environ["LIGER_FUSED_DECODE"] = fused
        os.environ["LIGER_LN_FOLD"] = "0"   # the fused pass reproduces the unfolded per-kernel path
        try:
            eng = LigerEngine(cfg, mode="serial", max_batch=4, max_seq=32, max_new=8, seed=0)
            bid = eng.submit(prompt.reshape(-1).astype(np.int32), 3, 20, 8, 0.0)
            eng.drain()
            _, toks = eng.poll(bid, want_tokens=True)
            st = eng.stats()
            eng.close()
        finally:
            os.environ.pop("LIGER_FUSED_DECODE", None)
            os.environ.pop("LIGER_LN_FOLD", None)
        out[fused] = toks
        assert st["gpu_launches"] > 0
    assert np.array_equal(out["1"], out["0"])   # fused (opt-in) and per-kernel engines agree
    ref, logits = om.greedy_generate(cfg, 0, prompt, 8, return_logits=True)
    ok = om.top2_margin(logits) > 0.02 * np.sqrt((logits ** 2).mean())
    for i in range(3):
        n = np.argmin(ok[i]) if not ok[i].all() else 8
        assert np.array_equal(out["1"][i, :n], ref[i, :n])
