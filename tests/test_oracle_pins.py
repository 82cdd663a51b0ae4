"""Pins of the fp64 oracle against things other than itself (CPU only).

Each pin is chosen so a plausible mistake (dropped term, wrong sign/index,
transposed operand) fails: an independent library implementation
(HF transformers OPT in fp64, torch layer_norm / gelu / SDPA), closed forms,
brute force on tiny inputs, and invariants the paper fixes (TP sharding and
decomposition change nothing; KV-cache decode = recompute).
"""
import json
import os

import numpy as np
import pytest
import torch

from liger_inputs import get_config, c0_uniform, bf16_rne, layer_activation
from oracle import model as om

GOLD = os.path.join(os.path.dirname(__file__), "golden")
TINY = get_config("tiny")


def test_c0_known_answers():
    rows = [l.split() for l in open(os.path.join(GOLD, "c0_known_answers.txt")) if l[0] != "#"]
    for seed, tid, idx, v in rows:
        got = c0_uniform(int(seed), int(tid), np.array([int(idx)]))[0]
        assert got == np.float32(v)


def test_bf16_rne_matches_torch():
    x = np.random.default_rng(0).standard_normal(10000).astype(np.float32) * 3
    ref = torch.from_numpy(x).to(torch.bfloat16).float().numpy()
    assert np.array_equal(bf16_rne(x), ref)


def test_layernorm_closed_forms_and_torch():
    rng = np.random.default_rng(1)
    g, b = rng.standard_normal(64), rng.standard_normal(64)
    const = np.full((3, 64), 2.5)
    assert np.allclose(om.layer_norm(const, g, b, 1e-5), b, atol=1e-12)   # constant row -> beta
    x = rng.standard_normal((5, 64)) * 4 + 1
    y = om.layer_norm(x, np.ones(64), np.zeros(64), 1e-5)
    assert np.allclose(y.mean(-1), 0, atol=1e-12)
    assert np.allclose(y.var(-1), 1 / (1 + 1e-5 / x.var(-1)), atol=1e-12)
    ref = torch.nn.functional.layer_norm(torch.from_numpy(x), (64,), torch.from_numpy(g),
                                         torch.from_numpy(b), 1e-5).numpy()
    assert np.allclose(om.layer_norm(x, g, b, 1e-5), ref, rtol=1e-12, atol=1e-12)


def test_gelu_relu_closed_forms():
    assert om.gelu_tanh(np.array(1.0)) == pytest.approx(0.8411919906082768, abs=1e-15)
    assert om.gelu_tanh(np.array(0.0)) == 0.0
    x = np.linspace(-6, 6, 1001)
    ref = torch.nn.functional.gelu(torch.from_numpy(x), approximate="tanh").numpy()
    assert np.allclose(om.gelu_tanh(x), ref, rtol=1e-13, atol=1e-15)
    assert np.array_equal(om.relu(np.array([-1.0, 0.0, 2.0])), [0.0, 0.0, 2.0])


def _brute_attention(q, k, v):
    """Direct exp, no max-subtraction, explicit loops (tiny shapes only)."""
    b, a, s, d = q.shape
    o = np.zeros_like(q)
    for bi in range(b):
        for h in range(a):
            for i in range(s):
                w = [np.exp(sum(q[bi, h, i, e] * k[bi, h, j, e] for e in range(d))) for j in range(i + 1)]
                z = sum(w)
                for e in range(d):
                    o[bi, h, i, e] = sum(w[j] * v[bi, h, j, e] for j in range(i + 1)) / z
    return o


def test_attention_brute_force_sdpa_and_special_cases():
    rng = np.random.default_rng(2)
    q, k, v = (rng.standard_normal((2, 2, 6, 4)) for _ in range(3))
    pos = np.arange(6)
    o = om.causal_attention(q, k, v, pos, pos)
    assert np.allclose(o, _brute_attention(q, k, v), rtol=1e-12, atol=1e-13)
    ref = torch.nn.functional.scaled_dot_product_attention(
        torch.from_numpy(q), torch.from_numpy(k), torch.from_numpy(v), is_causal=True, scale=1.0).numpy()
    assert np.allclose(o, ref, rtol=1e-12, atol=1e-13)
    # s = 1 -> o = v ; equal scores -> mean of visible V
    assert np.allclose(om.causal_attention(q[:, :, :1], k[:, :, :1], v[:, :, :1], pos[:1], pos[:1]), v[:, :, :1])
    oz = om.causal_attention(np.zeros_like(q), k, v, pos, pos)
    means = np.cumsum(v, axis=2) / (np.arange(6) + 1)[None, None, :, None]
    assert np.allclose(oz, means, atol=1e-13)


@pytest.mark.parametrize("t", [1, 2, 4])
def test_tp_sharded_equals_unsharded(t):
    w = om.layer_weights(TINY, 0, 0)
    x = layer_activation(TINY, 0, 0, 2 * 9).astype(np.float64).reshape(2, 9, TINY.hidden)
    ref, k, v = om.decoder_layer(TINY, w, x)
    got, kv = om.tp_decoder_layer(TINY, w, t, x)
    assert np.allclose(got, ref, rtol=1e-12, atol=1e-13)
    # the KV cache is head-sharded: concatenating the ranks' heads gives the full cache
    assert np.allclose(np.concatenate([kk for kk, _ in kv], axis=1), k, atol=1e-13)


def test_decomposition_equals_full():
    rng = np.random.default_rng(3)
    a, w, b = rng.standard_normal((7, 32)), rng.standard_normal((32, 48)), rng.standard_normal(48)
    full = a @ w + b
    for ks in ([8], [1] * 8, [2, 3, 3], [7, 1], [1, 2, 5]):
        assert np.allclose(om.gemm_decomposed(a, w, b, 8, ks), full, rtol=1e-13, atol=1e-13)
    parts = [rng.standard_normal((4, 16)) for _ in range(3)]
    for ks in ([8], [3, 5], [1] * 8):
        assert np.allclose(om.allreduce_decomposed(parts, 8, ks), sum(parts), atol=1e-14)
    with pytest.raises(AssertionError):
        om.gemm_decomposed(a, w, b, 8, [3, 3])       # a column not computed


def test_kv_cache_decode_equals_recompute():
    """P:316 KV cache: decode at step j equals the last row of a prefill over prompt + j tokens."""
    cfg = TINY
    w = om.layer_weights(cfg, 0, 1)
    x = layer_activation(cfg, 0, 1, 2 * 7).astype(np.float64).reshape(2, 7, cfg.hidden)
    _, k, v = om.decoder_layer(cfg, w, x[:, :5])
    step, _, _ = om.decoder_layer(cfg, w, x[:, 5:6], k, v, start_pos=5)
    full, _, _ = om.decoder_layer(cfg, w, x[:, :6])
    assert np.allclose(step[:, 0], full[:, 5], rtol=1e-12, atol=1e-13)


def _hf_opt(cfg, seed):
    from transformers import OPTConfig, OPTForCausalLM
    hc = OPTConfig(vocab_size=cfg.vocab, hidden_size=cfg.hidden, num_hidden_layers=cfg.n_layers,
                   ffn_dim=cfg.ffn, num_attention_heads=cfg.n_heads, max_position_embeddings=cfg.max_pos,
                   do_layer_norm_before=True, word_embed_proj_dim=cfg.hidden, dropout=0.0,
                   attention_dropout=0.0, activation_function="gelu_new" if cfg.act == "gelu_tanh" else "relu",
                   enable_bias=True, layer_norm_elementwise_affine=True, tie_word_embeddings=True,
                   pad_token_id=cfg.vocab - 1, bos_token_id=0, eos_token_id=1)
    hc._attn_implementation = "sdpa"   # eager upcasts softmax to fp32 (modeling_opt.py); SDPA stays fp64
    m = OPTForCausalLM(hc).double().eval()
    g = om.global_weights(cfg, seed)
    T = lambda a: torch.from_numpy(np.ascontiguousarray(a))
    dec = m.model.decoder
    with torch.no_grad():
        dec.embed_tokens.weight.copy_(T(g["e_tok"]))
        dec.embed_positions.weight.copy_(T(g["e_pos"]))
        dec.final_layer_norm.weight.copy_(T(g["lnf_g"]))
        dec.final_layer_norm.bias.copy_(T(g["lnf_b"]))
        h = cfg.hidden
        for l, layer in enumerate(dec.layers):
            w = om.layer_weights(cfg, seed, l)
            at = layer.self_attn
            at.q_proj.weight.copy_(T(w["w_qkv"][:, 0:h].T)); at.q_proj.bias.copy_(T(w["b_qkv"][0:h]))
            at.k_proj.weight.copy_(T(w["w_qkv"][:, h:2 * h].T)); at.k_proj.bias.copy_(T(w["b_qkv"][h:2 * h]))
            at.v_proj.weight.copy_(T(w["w_qkv"][:, 2 * h:].T)); at.v_proj.bias.copy_(T(w["b_qkv"][2 * h:]))
            at.out_proj.weight.copy_(T(w["w_o"].T)); at.out_proj.bias.copy_(T(w["b_o"]))
            layer.fc1.weight.copy_(T(w["w_1"].T)); layer.fc1.bias.copy_(T(w["b_1"]))
            layer.fc2.weight.copy_(T(w["w_2"].T)); layer.fc2.bias.copy_(T(w["b_2"]))
            layer.self_attn_layer_norm.weight.copy_(T(w["ln1_g"])); layer.self_attn_layer_norm.bias.copy_(T(w["ln1_b"]))
            layer.final_layer_norm.weight.copy_(T(w["ln2_g"])); layer.final_layer_norm.bias.copy_(T(w["ln2_b"]))
        m.lm_head.weight = dec.embed_tokens.weight
    return m


@pytest.mark.parametrize("act", ["gelu_tanh", "relu"])
def test_model_matches_hf_opt_fp64(act):
    """Library pin: HF transformers OPTForCausalLM (fp64, SDPA attention) with
    the same C0 weights gives the same logits and greedy tokens (tanh-GELU as
    configured for tiny/GLM-shaped, ReLU as in OPT)."""
    import dataclasses
    cfg = dataclasses.replace(TINY, act=act)
    m = _hf_opt(cfg, 0)
    prompt = np.random.default_rng(0).integers(0, cfg.vocab, size=(2, 32))
    toks, logits = om.greedy_generate(cfg, 0, prompt, 8, return_logits=True)
    with torch.no_grad():
        hf = m(torch.from_numpy(prompt)).logits[:, -1].numpy()
    assert np.allclose(logits[:, 0], hf, rtol=1e-10, atol=1e-12)
    with torch.no_grad():
        gen = m.generate(torch.from_numpy(prompt), max_new_tokens=8, do_sample=False,
                         attention_mask=torch.ones_like(torch.from_numpy(prompt)))
    assert np.array_equal(gen[:, 32:].numpy(), toks)


def test_top2_margin_hand_computed():
    """om.top2_margin (the near-tie gate of the token comparisons, reading R17) on
    hand-worked rows: the gap between the largest and the second-largest logit, a tie
    gives 0, order within the row does not matter, leading axes are kept."""
    from oracle import model as om
    x = np.array([[[1.0, 5.0, 3.0, -2.0], [0.5, 0.5, 0.1, 0.0]],
                  [[-1.0, -3.0, -0.25, -7.0], [2.0, 9.0, 9.0, 1.0]]])
    m = om.top2_margin(x)
    assert m.shape == (2, 2)
    assert np.array_equal(m, np.array([[2.0, 0.0], [0.75, 0.0]]))
    rng = np.random.default_rng(0)
    y = rng.standard_normal((3, 17))
    srt = -np.sort(-y, axis=-1)
    assert np.allclose(om.top2_margin(y[:, rng.permutation(17)]), srt[:, 0] - srt[:, 1])
