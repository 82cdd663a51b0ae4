"""Helpers shared by the GPU parity tests (test code only)."""
import numpy as np
import torch

from liger_inputs import KIND, weight_exp

BIAS_EXP = -6


def to_np64(t):
    return t.detach().float().cpu().numpy().astype(np.float64)


def bf16_dev(a, dev="cuda"):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(dev).bfloat16()


def errs(got, ref):
    """BASELINE.json metrics (R16): rel = max|g-r| / max|r|, MAE = mean|g-r|."""
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    d = np.abs(got - ref)
    return float(d.max() / max(np.abs(ref).max(), 1e-30)), float(d.mean())


def workspace(nbytes, dev="cuda"):
    return torch.zeros(max(int(nbytes), 16384) // 4 + 16, dtype=torch.int32, device=dev)


def shard_weights_device(L, cfg, seed, layer, t, r, dev="cuda"):
    """Build rank r's K-major shard of one layer on the device with the library's C0
    fill (the same layout liger_load_layer uses)."""
    h, f = cfg.hidden, cfg.ffn
    hl, fl = h // t, f // t
    tid = 16 * layer
    e = lambda *s: torch.empty(*s, dtype=torch.bfloat16, device=dev)
    W = dict(w_qkv=e(3 * hl, h), b_qkv=e(1, 3 * hl), w_o=e(h, hl), b_o=e(1, h), w_1=e(fl, h), b_1=e(1, fl),
             w_2=e(h, fl), b_2=e(1, h), ln1_g=e(1, h), ln1_b=e(1, h), ln2_g=e(1, h), ln2_b=e(1, h))
    for s in range(3):
        L.c0_fill(W["w_qkv"][s * hl:(s + 1) * hl], seed=seed, tensor_id=tid + KIND["w_qkv"],
                  row_off=s * h + r * hl, idx_row_stride=1, idx_col_stride=3 * h, exp=weight_exp(h))
        L.c0_fill(W["b_qkv"][:, s * hl:(s + 1) * hl], seed=seed, tensor_id=tid + KIND["b_qkv"],
                  col_off=s * h + r * hl, idx_row_stride=0, exp=BIAS_EXP)
    L.c0_fill(W["w_o"], seed=seed, tensor_id=tid + KIND["w_o"], col_off=r * hl, idx_row_stride=1,
              idx_col_stride=h, exp=weight_exp(h, "w_o"))
    L.c0_fill(W["b_o"], seed=seed, tensor_id=tid + KIND["b_o"], idx_row_stride=0, exp=BIAS_EXP)
    L.c0_fill(W["w_1"], seed=seed, tensor_id=tid + KIND["w_1"], row_off=r * fl, idx_row_stride=1,
              idx_col_stride=f, exp=weight_exp(h))
    L.c0_fill(W["b_1"], seed=seed, tensor_id=tid + KIND["b_1"], col_off=r * fl, idx_row_stride=0, exp=BIAS_EXP)
    L.c0_fill(W["w_2"], seed=seed, tensor_id=tid + KIND["w_2"], col_off=r * fl, idx_row_stride=1,
              idx_col_stride=h, exp=weight_exp(f, "w_2"))
    L.c0_fill(W["b_2"], seed=seed, tensor_id=tid + KIND["b_2"], idx_row_stride=0, exp=BIAS_EXP)
    for k, kind in (("ln1_g", 1), ("ln1_b", 2), ("ln2_g", 1), ("ln2_b", 2)):
        L.c0_fill(W[k], seed=seed, tensor_id=tid + KIND[k], idx_row_stride=0, kind=kind)
    return {k: (v.reshape(-1) if v.shape[0] == 1 else v) for k, v in W.items()}


def run_layer_rank(L, cfg, W, t, x, b, s, start_pos=0, kv=None, dev="cuda"):
    """One TP rank's share of a decoder layer through the C-ABI kernels:
    LN1 -> QKV(+bias, q scale) -> attention -> out-proj partial; then (after the
    caller sums the partials) the MLP half is done by run_mlp_rank."""
    h = cfg.hidden
    hl, al = h // t, cfg.n_heads // t
    d = h // cfg.n_heads
    M = x.shape[0]
    y = torch.empty_like(x)
    L.add_layernorm(x, W["ln1_g"], W["ln1_b"], y, eps=cfg.ln_eps)
    qkv = torch.empty(M, 3 * hl, dtype=torch.bfloat16, device=dev)
    ws = workspace(L.gemm_workspace_bytes(M, 3 * hl, h))
    L.gemm(y, W["w_qkv"], qkv, bias=W["b_qkv"], scale_cols=hl, scale=1.0 / d ** 0.5, workspace=ws)
    o = torch.empty(M, hl, dtype=torch.bfloat16, device=dev)
    if kv is None:
        maxp = (s + 15) // 16 + 1
        pool = torch.zeros(b * maxp, 2, al, 16, d, dtype=torch.bfloat16, device=dev)
        pt = torch.arange(b * maxp, dtype=torch.int32, device=dev).reshape(b, maxp)
        kv = (pool, pt)
        L.attn_prefill(qkv, o, pool, pt, b=b, s=s, heads=al, d=d)
    else:
        pool, pt = kv
        aw = workspace(L.attn_decode_workspace_bytes(b, al, d, start_pos + 1))
        L.attn_decode(qkv, o, pool, pt, b=b, pos=start_pos, heads=al, d=d, workspace=aw)
    part = torch.empty(M, h, dtype=torch.bfloat16, device=dev)
    ws2 = workspace(L.gemm_workspace_bytes(M, h, hl))
    L.gemm(o, W["w_o"], part, workspace=ws2)
    return part, kv


def run_mlp_rank(L, cfg, W, t, y2, dev="cuda"):
    h, fl = cfg.hidden, cfg.ffn // t
    M = y2.shape[0]
    hb = torch.empty(M, fl, dtype=torch.bfloat16, device=dev)
    L.gemm(y2, W["w_1"], hb, bias=W["b_1"], act=cfg.act, workspace=workspace(L.gemm_workspace_bytes(M, fl, h)))
    part = torch.empty(M, h, dtype=torch.bfloat16, device=dev)
    L.gemm(hb, W["w_2"], part, workspace=workspace(L.gemm_workspace_bytes(M, h, fl)))
    return part
