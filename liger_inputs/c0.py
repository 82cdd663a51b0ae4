"""C0: seeded counter-based weight generator (SURVEY.md §8(c) "C0 details").

BASELINE.json asks for "identical seeded random weights" on the oracle and the
GPU path without shared code.  Both sides therefore implement this exact
definition independently (this numpy version; `c0_fill_kernel` in `csrc/norm.cu` on the device):

    x   = seed*0x9E3779B97F4A7C15 + tensor_id*0xD1B54A32D192ED03 + idx + 0x9E3779B97F4A7C15   (mod 2^64)
    u   = mix64(x)     (SplitMix64 finaliser)
    r   = int(u >> 40) - 2^23                 (24-bit signed integer)
    v   = r * 2^-23                           in [-1, 1), exact in fp32
    w   = bf16_rne(f32(v * 2^e))              (power-of-two scale: exact)
    gamma = bf16_rne(f32(1 + f32(v * 2^-4))), beta = bf16_rne(v * 2^-4)

`idx` is the row-major index in the UNSHARDED logical [K_in, N_out] matrix
(k*N + n) or the element index of a vector; a tensor-parallel shard generates
its elements from their global indices.

Scales (reading R16, chosen to keep per-layer output RMS well below
1 so that bf16 output rounding stays inside BASELINE.json's MAE bound):
  GEMM weight with fan-in K : e = round(0.5*log2(3/K)) - 1   (W_qkv, W_1)
                              e = round(0.5*log2(3/K)) - 2   (output projections W_o, W_2,
                                  halving the residual-branch gain, as GPT-2 scales them)
  bias                      : e = -6
  embeddings E_tok, E_pos   : e = round(-0.5*log2(h)) - 1   (emb_exp(h): RMS ~ 0.3/sqrt(h),
                                  small against the layers' output so that the decoder
                                  layers decide the tied head's argmax -- the self term
                                  E[tok].E[tok] grows like sqrt(h) against the others; with
                                  a fixed 2^-3 a model with zero layers gave the same greedy
                                  tokens; R16)
  layer-input activations   : e = -2   (layer-level parity tests only)
"""
import math
import numpy as np

M64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15
TMUL = 0xD1B54A32D192ED03

KIND = {
    "w_qkv": 0, "b_qkv": 1, "w_o": 2, "b_o": 3, "w_1": 4, "b_1": 5,
    "w_2": 6, "b_2": 7, "ln1_g": 8, "ln1_b": 9, "ln2_g": 10, "ln2_b": 11,
}
GLOBAL_ID = {"e_tok": 0xFFFF00, "e_pos": 0xFFFF01, "lnf_g": 0xFFFF02, "lnf_b": 0xFFFF03}
ACT_ID_BASE = 0xFFFF10   # + layer: activations for per-layer parity tests

BIAS_EXP = -6
ACT_EXP = -2


def mix64(x: np.ndarray) -> np.ndarray:
    """SplitMix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = x ^ (x >> np.uint64(30))
        x = x * np.uint64(0xBF58476D1CE4E5B9)
        x = x ^ (x >> np.uint64(27))
        x = x * np.uint64(0x94D049BB133111EB)
        x = x ^ (x >> np.uint64(31))
    return x


def c0_uniform(seed: int, tensor_id: int, idx: np.ndarray) -> np.ndarray:
    """v in [-1,1) as float32 (exact: 24 significant bits)."""
    base = (seed * GOLDEN + tensor_id * TMUL + GOLDEN) & M64
    idx = np.asarray(idx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = idx + np.uint64(base)
    u = mix64(x)
    r = (u >> np.uint64(40)).astype(np.int64) - (1 << 23)
    return (r.astype(np.float32) * np.float32(2.0 ** -23)).astype(np.float32)


def bf16_rne(f: np.ndarray) -> np.ndarray:
    """Round float32 -> bfloat16 (round to nearest even) via bits; returned as float32."""
    f = np.ascontiguousarray(f, dtype=np.float32)
    u = f.view(np.uint32).astype(np.uint64)
    u = u + np.uint64(0x7FFF) + ((u >> np.uint64(16)) & np.uint64(1))
    u = (u & np.uint64(0xFFFF0000)).astype(np.uint32)
    return u.view(np.float32)


OUT_PROJ = ("w_o", "w_2")


def weight_exp(k_in: int, kind: str = "w_qkv") -> int:
    """Round half to even (Python round); the CUDA side uses nearbyint."""
    return int(round(0.5 * math.log2(3.0 / k_in))) - (2 if kind in OUT_PROJ else 1)


def emb_exp(hidden: int) -> int:
    """Scale exponent of the embeddings E_tok / E_pos (round half to even; CUDA: nearbyint)."""
    return int(round(-0.5 * math.log2(hidden))) - 1


def c0_values(seed: int, tensor_id: int, idx: np.ndarray, exp: int) -> np.ndarray:
    v = c0_uniform(seed, tensor_id, idx)
    return bf16_rne(v * np.float32(2.0 ** exp))


def _gamma(seed, tid, idx):
    v = c0_uniform(seed, tid, idx)
    return bf16_rne(np.float32(1.0) + v * np.float32(2.0 ** -4))


def _beta(seed, tid, idx):
    v = c0_uniform(seed, tid, idx)
    return bf16_rne(v * np.float32(2.0 ** -4))


def layer_tensor_shape(cfg, kind: str):
    h, f = cfg.hidden, cfg.ffn
    return {
        "w_qkv": (h, 3 * h), "b_qkv": (3 * h,), "w_o": (h, h), "b_o": (h,),
        "w_1": (h, f), "b_1": (f,), "w_2": (f, h), "b_2": (h,),
        "ln1_g": (h,), "ln1_b": (h,), "ln2_g": (h,), "ln2_b": (h,),
    }[kind]


def layer_tensor(cfg, seed: int, layer: int, kind: str, cols=None, rows=None) -> np.ndarray:
    """Logical (unsharded) layer tensor as float32 holding bf16 values.

    Matrices are [K_in, N_out] (y = x @ W).  `cols` / `rows` optionally select a
    subset of N / K indices (generated from their global indices)."""
    tid = 16 * layer + KIND[kind]
    shape = layer_tensor_shape(cfg, kind)
    if len(shape) == 2:
        K, N = shape
        r = np.arange(K, dtype=np.uint64) if rows is None else np.asarray(rows, dtype=np.uint64)
        c = np.arange(N, dtype=np.uint64) if cols is None else np.asarray(cols, dtype=np.uint64)
        idx = r[:, None] * np.uint64(N) + c[None, :]
        return c0_values(seed, tid, idx, weight_exp(K, kind))
    n = shape[0]
    idx = np.arange(n, dtype=np.uint64) if cols is None else np.asarray(cols, dtype=np.uint64)
    if kind.endswith("_g"):
        return _gamma(seed, tid, idx)
    if kind in ("ln1_b", "ln2_b"):
        return _beta(seed, tid, idx)
    return c0_values(seed, tid, idx, BIAS_EXP)


def global_tensor(cfg, seed: int, kind: str, rows=None) -> np.ndarray:
    tid = GLOBAL_ID[kind]
    h = cfg.hidden
    if kind in ("e_tok", "e_pos"):
        nrows = cfg.vocab if kind == "e_tok" else cfg.max_pos + 2
        r = np.arange(nrows, dtype=np.uint64) if rows is None else np.asarray(rows, dtype=np.uint64)
        idx = r[:, None] * np.uint64(h) + np.arange(h, dtype=np.uint64)[None, :]
        return c0_values(seed, tid, idx, emb_exp(h))
    idx = np.arange(h, dtype=np.uint64)
    return _gamma(seed, tid, idx) if kind == "lnf_g" else _beta(seed, tid, idx)


def layer_activation(cfg, seed: int, layer: int, m: int) -> np.ndarray:
    """Synthetic bf16 layer input x [m, h] for per-layer parity tests."""
    idx = np.arange(m * cfg.hidden, dtype=np.uint64).reshape(m, cfg.hidden)
    return c0_values(seed, ACT_ID_BASE + layer, idx, ACT_EXP)
