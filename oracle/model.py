"""Plain fp64 forward of the decoder layer and model (oracle; test infrastructure only).

The paper never writes the layer math out: it reuses FasterTransformer kernels
(§4) and Megatron intra-op partitioning with "two all-reduce
synchronizations ... in each transformer layer".  Liger changes WHEN
kernels run, never WHAT they compute (interleaving; decomposition into
kernels "with equal capabilities").  So this oracle is the plain
definition of an OPT-style pre-LN decoder (reading R13):

  C1  x0   = E_tok[id] + E_pos[pos + 2]
  C2  LN(x) = (x - mean) / sqrt(var + eps) * g + b     (population variance)
  C3  [q|k|v] = LN1(x) @ W_qkv + b_qkv ;  q *= d^-1/2   (after the bias)
  C4  o = softmax_j(q.k_j, j <= pos(i)) @ V             (per head, causal)
  C5  x1 = x + o @ W_o + b_o
  C6  x2 = x1 + act(LN2(x1) @ W_1 + b_1) @ W_2 + b_2
  C7  logits = LN_f(x_L) @ E_tok^T ; token = argmax (lowest index on ties)
  C8  TP emulation: rank r owns heads [r a/t, (r+1) a/t) of q/k/v, the same rows
      of W_o, columns [r f/t, (r+1) f/t) of W_1/b_1 and those rows of W_2;
      partials are summed (the all-reduce) and b_o / b_2 added once.
  C9  decomposition (Fig. 9 "vertical"): the k/F piece of a GEMM is
      the column block [c0, c0 + k N/F) of W; the concatenation of the pieces
      is the full product.

Everything is float64; matmul is numpy's (a library primitive as one step).
"""
import numpy as np

from liger_inputs import layer_tensor, global_tensor

F64 = np.float64


# ---------------------------------------------------------------- primitives
def layer_norm(x, g, b, eps):
    """C2.  Population variance, eps inside the sqrt (reading R26)."""
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps) * g + b


def gelu_tanh(x):
    return 0.5 * x * (1.0 + np.tanh(np.sqrt(2.0 / np.pi) * (x + 0.044715 * x ** 3)))


def relu(x):
    return np.maximum(x, 0.0)


def activation(cfg):
    return relu if cfg.act == "relu" else gelu_tanh


def softmax(s, axis=-1):
    m = s.max(axis=axis, keepdims=True)
    e = np.exp(s - m)
    return e / e.sum(axis=axis, keepdims=True)


def causal_attention(q, k, v, q_pos, k_pos):
    """C4.  q [b, a, s, d] (already scaled); k, v [b, a, ctx, d];
    q_pos [s], k_pos [ctx] absolute positions.  Key j visible to query i iff
    k_pos[j] <= q_pos[i]."""
    s = np.einsum("bhid,bhjd->bhij", q, k)
    mask = k_pos[None, :] <= q_pos[:, None]
    s = np.where(mask[None, None], s, -np.inf)
    p = softmax(s, axis=-1)
    return np.einsum("bhij,bhjd->bhid", p, v)


# ---------------------------------------------------------------- weights
LAYER_KINDS = ("w_qkv", "b_qkv", "w_o", "b_o", "w_1", "b_1", "w_2", "b_2",
               "ln1_g", "ln1_b", "ln2_g", "ln2_b")


def layer_weights(cfg, seed, layer):
    """All tensors of one layer, logical [K_in, N_out] layout, float64."""
    return {k: layer_tensor(cfg, seed, layer, k).astype(F64) for k in LAYER_KINDS}


def global_weights(cfg, seed):
    return {k: global_tensor(cfg, seed, k).astype(F64) for k in ("e_tok", "e_pos", "lnf_g", "lnf_b")}


# ---------------------------------------------------------------- one layer
def _split_heads(t, a):
    b, s, n = t.shape
    return t.reshape(b, s, a, n // a).transpose(0, 2, 1, 3)


def _merge_heads(t):
    b, a, s, d = t.shape
    return t.transpose(0, 2, 1, 3).reshape(b, s, a * d)


def attention_block(cfg, w, x, past_k=None, past_v=None, start_pos=0):
    """LN1 -> QKV -> attention.  Returns (o [b,s,h] concat heads, k_all, v_all)."""
    h, a = cfg.hidden, cfg.n_heads
    d = h // a
    y = layer_norm(x, w["ln1_g"], w["ln1_b"], cfg.ln_eps)
    qkv = y @ w["w_qkv"] + w["b_qkv"]
    q = qkv[..., 0:h] * (d ** -0.5)
    k = qkv[..., h:2 * h]
    v = qkv[..., 2 * h:3 * h]
    q, k, v = _split_heads(q, a), _split_heads(k, a), _split_heads(v, a)
    if past_k is not None:
        k = np.concatenate([past_k, k], axis=2)
        v = np.concatenate([past_v, v], axis=2)
    s = x.shape[1]
    q_pos = np.arange(start_pos, start_pos + s)
    k_pos = np.arange(k.shape[2])
    o = causal_attention(q, k, v, q_pos, k_pos)
    return _merge_heads(o), k, v


def decoder_layer(cfg, w, x, past_k=None, past_v=None, start_pos=0):
    """C3-C6 for one unsharded layer.  x [b, s, h] float64.
    Returns (x2, k_all, v_all) with k_all/v_all [b, a, ctx, d] (the KV cache)."""
    o, k, v = attention_block(cfg, w, x, past_k, past_v, start_pos)
    x1 = x + o @ w["w_o"] + w["b_o"]
    y2 = layer_norm(x1, w["ln2_g"], w["ln2_b"], cfg.ln_eps)
    x2 = x1 + activation(cfg)(y2 @ w["w_1"] + w["b_1"]) @ w["w_2"] + w["b_2"]
    return x2, k, v


# ---------------------------------------------------------------- TP (C8)
def shard_layer(cfg, w, t, r):
    """Rank r's shard of one layer's weights under Megatron TP degree t."""
    h, a, f = cfg.hidden, cfg.n_heads, cfg.ffn
    d = h // a
    assert a % t == 0 and f % t == 0
    c0, c1 = r * (a // t) * d, (r + 1) * (a // t) * d
    f0, f1 = r * f // t, (r + 1) * f // t
    cols = np.r_[c0:c1, h + c0:h + c1, 2 * h + c0:2 * h + c1]
    return {
        "w_qkv": w["w_qkv"][:, cols], "b_qkv": w["b_qkv"][cols],
        "w_o": w["w_o"][c0:c1, :],
        "w_1": w["w_1"][:, f0:f1], "b_1": w["b_1"][f0:f1],
        "w_2": w["w_2"][f0:f1, :],
        "ln1_g": w["ln1_g"], "ln1_b": w["ln1_b"], "ln2_g": w["ln2_g"], "ln2_b": w["ln2_b"],
    }


def tp_partials_attn(cfg, ws, t, x, start_pos=0, past=None):
    """Per-rank row-parallel partials of the out-projection (before all-reduce #1)."""
    a_loc = cfg.n_heads // t
    parts, kv = [], []
    for r in range(t):
        w = ws[r]
        sub = _LocalCfg(cfg, t)
        pk, pv = (None, None) if past is None else past[r]
        o, k, v = attention_block(sub, w, x, pk, pv, start_pos)
        parts.append(o @ w["w_o"])
        kv.append((k, v))
    assert all(p.shape[-1] == cfg.hidden for p in parts) and a_loc * t == cfg.n_heads
    return parts, kv


def tp_partials_mlp(cfg, ws, t, y2):
    act = activation(cfg)
    return [act(y2 @ ws[r]["w_1"] + ws[r]["b_1"]) @ ws[r]["w_2"] for r in range(t)]


class _LocalCfg:
    """Per-rank view for attention_block: a/t heads of width d.  attention_block
    normalises the full-width x with the replicated LN1 weights, then slices the
    rank's 3h/t QKV columns as [q | k | v] of width h/t each."""

    def __init__(self, cfg, t):
        self.hidden = cfg.hidden // t
        self.n_heads = cfg.n_heads // t
        self.ln_eps = cfg.ln_eps


def tp_decoder_layer(cfg, w, t, x, start_pos=0, past=None, allreduce=None):
    """C8: TP-emulated layer.  `allreduce(list_of_partials) -> sum` defaults to a
    plain sum over ranks; a gloo test passes a real collective."""
    ws = [shard_layer(cfg, w, t, r) for r in range(t)]
    red = allreduce or (lambda ps: np.sum(ps, axis=0))
    parts, kv = tp_partials_attn(cfg, ws, t, x, start_pos, past)
    x1 = x + red(parts) + w["b_o"]
    y2 = layer_norm(x1, w["ln2_g"], w["ln2_b"], cfg.ln_eps)
    x2 = x1 + red(tp_partials_mlp(cfg, ws, t, y2)) + w["b_2"]
    return x2, kv


# ---------------------------------------------------------------- decomposition (C9)
def gemm_piece(a, w, bias, c0, c1):
    """The vertical piece [c0, c1) of a @ w + bias (Fig. 9)."""
    out = a @ w[:, c0:c1]
    return out if bias is None else out + bias[c0:c1]


def gemm_decomposed(a, w, bias, F, ks):
    """Run a GEMM as consecutive pieces of ks[i]/F of its N columns and concatenate.
    sum(ks) must equal F (each column computed exactly once)."""
    N = w.shape[1]
    assert sum(ks) == F and N % F == 0
    step = N // F
    outs, c = [], 0
    for k in ks:
        outs.append(gemm_piece(a, w, bias, c * step, (c + k) * step))
        c += k
    return np.concatenate(outs, axis=-1)


def allreduce_decomposed(parts, F, ks):
    """All-reduce issued as contiguous chunks of ks[i]/F of the elements."""
    flat = [p.reshape(-1) for p in parts]
    n = flat[0].size
    assert sum(ks) == F and n % F == 0
    step = n // F
    out, c = np.empty(n), 0
    for k in ks:
        sl = slice(c * step, (c + k) * step)
        out[sl] = np.sum([f[sl] for f in flat], axis=0)
        c += k
    return out.reshape(parts[0].shape)


# ---------------------------------------------------------------- full model (C1, C7)
def embed(cfg, g, ids, positions):
    """C1: OPT learned positions with offset 2."""
    return g["e_tok"][ids] + g["e_pos"][positions + 2]


def lm_head(cfg, g, x_last):
    """C7: final LN, tied head (no bias).  Returns logits [b, V]."""
    y = layer_norm(x_last, g["lnf_g"], g["lnf_b"], cfg.ln_eps)
    return y @ g["e_tok"].T


def greedy_generate(cfg, seed, prompt, n_new, layers=None, g=None, return_logits=False, return_hidden=False):
    """Greedy generation with a KV cache (reading R22).

    prompt int [b, s].  Pass 0 is the prefill over the prompt and yields token 1;
    pass j (1 <= j < n_new) feeds token j at position s + j - 1 (M = b) and
    yields token j+1.  Returns tokens [b, n_new] (and per-pass logits [b, n_new, V];
    with return_hidden also the LM-head input x_L of the last token [b, n_new, h])."""
    layers = layers or [layer_weights(cfg, seed, l) for l in range(cfg.n_layers)]
    g = g or global_weights(cfg, seed)
    b, s = prompt.shape
    x = embed(cfg, g, prompt, np.arange(s))
    cache = []
    for l, w in enumerate(layers):
        x, k, v = decoder_layer(cfg, w, x, start_pos=0)
        cache.append((k, v))
    logits = [lm_head(cfg, g, x[:, -1])]
    hidden = [x[:, -1]]
    toks = [np.argmax(logits[-1], axis=-1)]
    for j in range(1, n_new):
        pos = s + j - 1
        x = embed(cfg, g, toks[-1][:, None], np.array([pos]))
        for l, w in enumerate(layers):
            x, k, v = decoder_layer(cfg, w, x, cache[l][0], cache[l][1], start_pos=pos)
            cache[l] = (k, v)
        logits.append(lm_head(cfg, g, x[:, -1]))
        hidden.append(x[:, -1])
        toks.append(np.argmax(logits[-1], axis=-1))
    out = np.stack(toks, axis=1)
    if return_hidden:
        return out, np.stack(logits, axis=1), np.stack(hidden, axis=1)
    return (out, np.stack(logits, axis=1)) if return_logits else out


def top2_margin(logits):
    """Gap between the largest and second-largest logit per row (reading R17)."""
    srt = np.sort(logits, axis=-1)
    return srt[..., -1] - srt[..., -2]
