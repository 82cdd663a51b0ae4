"""Dev: where the t = 1 two-stream capacity run spends its time (in-kernel %globaltimer
trace of every CTA: kind, SM, entry, PDL-wait release, exit).

    python tools/timeline_capacity.py [n_batches] [mode]

Serves n_batches (default 4) of bench.py's mixed workload (b in {2,4,8}, prompt
U[128,512], 32 generated tokens) all offered at once, OPT-13B TP = 1, and prints, over
the traced span: per kernel kind the SM-time share (sum of release->exit over CTAs /
(148 x span)), the wall-time coverage (time at least one CTA of the kind works), and the
coverage of 'no GEMM working' (neither stream streams weights)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from liger_inputs import get_config, make_trace
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine

KIND = {1: "gemm", 2: "fixup", 3: "attn_dec", 4: "attn_pre", 5: "add_ln", 6: "embed", 7: "argmax", 8: "pick",
        9: "fused"}


def coverage(iv):
    """Total length of the union of intervals iv [(a, b)]."""
    if len(iv) == 0:
        return 0.0
    iv = iv[np.argsort(iv[:, 0])]
    tot, ca, cb = 0.0, iv[0, 0], iv[0, 1]
    for a, b in iv[1:]:
        if a > cb:
            tot += cb - ca
            ca, cb = a, b
        elif b > cb:
            cb = b
    return tot + cb - ca


def main():
    nb = int(sys.argv[1]) if len(sys.argv) > 1 else 4
    mode = sys.argv[2] if len(sys.argv) > 2 else "interleaved"
    cfg = get_config("opt-13b")
    eng = LigerEngine(cfg, mode=mode, max_batch=8, max_seq=512, max_new=32, max_inflight=2, seed=0)
    warm = make_trace(2, float("inf"), seed=5, vocab=cfg.vocab, n_decode=32)
    for r in warm:
        eng.submit(r["tokens"], r["batch"], r["seq_len"], r["n_decode"], 0.0)
    eng.drain()
    trace = make_trace(nb, float("inf"), seed=0, vocab=cfg.vocab, n_decode=32)
    cap = 1 << 23
    torch.cuda.synchronize()
    L.trace_start(cap)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for r in trace:
        eng.submit(r["tokens"], r["batch"], r["seq_len"], r["n_decode"], 0.0)
    eng.drain()
    e1.record()
    torch.cuda.synchronize()
    rec = L.trace_stop(cap)
    ms = e0.elapsed_time(e1)
    print(f"mode {mode}: {nb} batches {[r['batch'] for r in trace]} x prompts {[r['seq_len'] for r in trace]}: "
          f"{ms:.1f} ms, {len(rec)} CTA records (cap {cap})")
    t0 = rec["t0"].min()
    span = float(rec["t2"].max() - t0)
    w = np.stack([(rec["t1"] - t0).astype(np.float64), (rec["t2"] - t0).astype(np.float64)], 1)
    nsm = int(rec["smid"].max()) + 1
    print(f"traced span {span / 1e3:.1f} us over {nsm} SMs")
    print(f"{'kind':>10} {'CTAs':>9} {'SM-time share':>14} {'wall coverage':>14}")
    for k in np.unique(rec["kid"]):
        m = rec["kid"] == k
        smt = float((w[m, 1] - w[m, 0]).sum())
        print(f"{KIND.get(int(k), k):>10} {int(m.sum()):>9} {smt / (nsm * span):>14.3f} "
              f"{coverage(w[m]) / span:>14.3f}")
    g = rec["kid"] == 1
    print(f"no GEMM CTA working: {1 - coverage(w[g]) / span:.3f} of the span")
    # how many GEMM CTAs work concurrently (event sweep, time-weighted)
    ev = np.concatenate([w[g, 0], w[g, 1]])
    dv = np.concatenate([np.ones(int(g.sum())), -np.ones(int(g.sum()))])
    o = np.argsort(ev, kind="stable")
    ev, dv = ev[o], dv[o]
    cnt = np.cumsum(dv)[:-1]
    dt = np.diff(ev)
    b = np.minimum(cnt.astype(int) // 37, 8)
    hist = np.bincount(b, weights=dt, minlength=9) / span
    print("GEMM CTAs working concurrently (fraction of span): " +
          ", ".join(f"[{37 * i},{37 * (i + 1)}): {hist[i]:.3f}" for i in range(9) if hist[i] > 0.001))
    eng.close()


if __name__ == "__main__":
    main()
