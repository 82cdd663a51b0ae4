"""Dev: per-phase timeline of the fused decode pass (csrc/decode_fused.cu) from the
in-kernel %globaltimer trace: for the last decode pass of one OPT-13B TP=1 batch,
per phase (layer, LN1/QKV/ATTN/OUT/LN2/FC1/FC2): first CTA start, median / last
CTA "share done", last signal -- relative to the pass start, in us.

    python tools/fused_timeline.py [b] [layers_to_print]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from liger_inputs import get_config
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine

b = int(sys.argv[1]) if len(sys.argv) > 1 else 8
nprint = int(sys.argv[2]) if len(sys.argv) > 2 else 2
cfg = get_config("opt-13b")
eng = LigerEngine(cfg, mode="serial", max_batch=8, max_seq=512, max_new=32, seed=0)
toks = torch.from_numpy(np.random.default_rng(0).integers(0, cfg.vocab, size=b * 256).astype(np.int32)).cuda()
eng.submit(None, b, 256, 3, 0.0, device_tokens=toks); eng.drain()
torch.cuda.synchronize()
L.trace_start(1 << 21)
eng.submit(None, b, 256, 3, 0.0, device_tokens=toks); eng.drain()
torch.cuda.synchronize()
rec = L.trace_stop(1 << 21)
ph = rec[(rec["kid"] >= 0x200) & (rec["kid"] < 0x210)]
NL = cfg.n_layers
per = 7 * NL
names = ["LN1", "QKV", "ATTN", "OUT", "LN2", "FC1", "FC2"]
ctas = np.unique(ph["cta"])
rows = []   # [cta][j] -> (t0, t1, t2)
for c in ctas:
    r = ph[ph["cta"] == c]
    r = r[np.argsort(r["t0"])][-per:]
    rows.append(r)
A = np.stack([np.stack([r["t0"], r["t1"], r["t2"]], 1) for r in rows]).astype(np.int64)   # [G, per, 3]
T0 = A[:, 0, 0].min()
print(f"{len(ctas)} CTAs; pass = {(A[:, -1, 2].max() - T0) / 1e3:.1f} us")
print(f"{'phase':>10} {'start':>8} {'done_med':>8} {'done_max':>8} {'signal':>8} {'dur':>7}")
prev = T0
tot = {n: 0.0 for n in names}
for j in range(per):
    l, p = divmod(j, 7)
    t0 = A[:, j, 0].min(); dmed = np.median(A[:, j, 1]); dmax = A[:, j, 1].max(); sig = A[:, j, 2].max()
    tot[names[p]] += (sig - prev) / 1e3
    if l < nprint or l == NL - 1:
        print(f"{l:3d} {names[p]:>6} {(t0 - T0) / 1e3:8.2f} {(dmed - T0) / 1e3:8.2f} {(dmax - T0) / 1e3:8.2f} "
              f"{(sig - T0) / 1e3:8.2f} {(sig - prev) / 1e3:7.2f}")
    prev = sig
print("per-phase totals (us/pass):", {k: round(v, 1) for k, v in tot.items()})

# per-unit accumulator-ready times of layer 1's GEMMs, relative to that layer's LN1 signal
un = rec[(rec["kid"] >= 0x300) & (rec["kid"] < 0x304)]
for g, nm in enumerate(["QKV", "OUT", "FC1", "FC2"]):
    u = un[un["kid"] == 0x300 + g]
    # the last pass: per CTA, the last NL*k records; take layer 1 -> use time window of layer 1 phases
    j = 7 * 1 + [1, 3, 5, 6][g]
    lo = A[:, j - 1, 2].max(); hi = A[:, j, 2].max()
    sel = u[(u["t2"] >= lo) & (u["t2"] <= hi + 1000)]
    if len(sel) == 0:
        continue
    per_cta = {}
    for x in sel:
        per_cta.setdefault(int(x["cta"]), []).append((x["t0"] - lo) / 1e3)
    cnt = np.array([len(v) for v in per_cta.values()])
    last = np.array([max(v) for v in per_cta.values()])
    first = np.array([min(v) for v in per_cta.values()])
    print(f"L1 {nm}: units/CTA min {cnt.min()} max {cnt.max()}; first unit wait-start median {np.median(first):.1f}; "
          f"acc-ready of last unit: median {np.median(last):.1f} max {last.max():.1f} us after phase k-1 signal")
    order = np.argsort(last)[::-1][:3]
    ks = list(per_cta.keys())
    for o in order:
        print("   slow CTA", ks[o], "unit ready times", [round(v, 1) for v in sorted(per_cta[ks[o]])])
    sel2 = sel[np.argsort(sel["t2"])]
    print("   ready (t2) deciles:", [round((np.percentile(sel2["t2"], q) - lo) / 1e3, 1) for q in (10, 50, 90, 100)])

# intra-phase breakdown (layer 1 window), relative to the previous phase's global signal
def win(j):
    return A[:, j - 1, 2].max(), A[:, j, 2].max()
for kid, j, nm, cols in [(0x400, 7, "LN1 rows", ("wait released", "rows done", "signalled")),
                         (0x400, 11, "LN2 rows", ("wait released", "rows done", "signalled")),
                         (0x430, 9, "ATTN", ("items done", "merges done", "signalled")),
                         (0x410, 8, "QKV", ("units done", "published", "")), (0x420, 8, "QKV", ("", "reduced", "signalled")),
                         (0x410, 12, "FC1", ("units done", "published", "")), (0x420, 12, "FC1", ("", "reduced", "signalled")),
                         (0x413, 13, "FC2", ("units done", "published", "")), (0x423, 13, "FC2", ("", "reduced", "signalled"))]:
    lo, hi = win(j)
    r = rec[(rec["kid"] == kid) & (rec["t2"] >= lo - 1000) & (rec["t2"] <= hi + 2000)]
    if len(r) == 0:
        continue
    f = lambda a: f"med {np.median((a.astype(np.int64) - lo) / 1e3):6.1f} max {((a.astype(np.int64) - lo).max()) / 1e3:6.1f}"
    print(f"{nm:9s} n={len(r):3d}  {cols[0]:>13}: {f(r['t0'])} | {cols[1]:>11}: {f(r['t1'])} | {cols[2]:>10}: {f(r['t2'])}")
