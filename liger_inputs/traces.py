"""Synthetic request traces.

The paper serves 2000 requests at a constant, rising arrival rate with random
sequence lengths 16-128 and batch sizes 2/4/8.  BASELINE.json
asks for Poisson traces with prompt 128-512 and 32 decode tokens (OPT) or
prompt 2048 (GLM-shaped).  One trace entry is one pre-packed batch
(reading R12: "request" = one batch of b equal-length sequences).
"""
import numpy as np


def make_trace(n_batches: int, rate_per_s: float, seed: int = 0, *, batch_sizes=(2, 4, 8),
               prompt_range=(128, 512), n_decode: int = 32, vocab: int = 50272,
               poisson: bool = True):
    """Return a list of dicts {arrival_s, batch, seq_len, n_decode, tokens[int32 b*s]}.

    Inter-arrival ~ Exp(1/rate) (Poisson) or constant 1/rate (the paper's
    constant-rate variant, reading R21).  rate_per_s = inf => all arrive at 0."""
    rng = np.random.default_rng(seed)
    out = []
    t = 0.0
    for i in range(n_batches):
        if i > 0 and np.isfinite(rate_per_s):
            t += rng.exponential(1.0 / rate_per_s) if poisson else 1.0 / rate_per_s
        b = int(rng.choice(np.asarray(batch_sizes)))
        lo, hi = prompt_range
        s = int(rng.integers(lo, hi + 1))
        toks = rng.integers(0, vocab, size=b * s, dtype=np.int64).astype(np.int32)
        out.append(dict(arrival_s=float(t), batch=b, seq_len=s, n_decode=int(n_decode), tokens=toks))
    return out
