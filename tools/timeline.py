"""Dev: per-launch timeline of decode passes from the in-kernel %globaltimer trace.

    python tools/timeline.py [b] [n_layers_to_print]

Serves one OPT-13B TP=1 batch (b x 256 prompt, 3 generated tokens) and prints, for
the last decode pass, every kernel launch in order: CTA count, first entry, PDL-wait
release (min / max over CTAs), last exit, relative to the pass start (us), plus a
per-kind summary over the pass (sum of first-entry-to-last-exit spans and gaps)."""
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
eng.submit(None, b, 256, 3, 0.0, device_tokens=toks); eng.drain()      # warm
torch.cuda.synchronize()
L.trace_start(1 << 21)
eng.submit(None, b, 256, 3, 0.0, device_tokens=toks); eng.drain()
torch.cuda.synchronize()
rec = L.trace_stop(1 << 21)
print(f"{len(rec)} CTA records")

launches = []
for kid in np.unique(rec["kid"]):
    r = rec[rec["kid"] == kid]
    r = r[np.argsort(r["t0"], kind="stable")]
    seen, cur = set(), []
    for x in r:
        if x["cta"] in seen:
            launches.append((kid, cur)); seen, cur = set(), []
        seen.add(x["cta"]); cur.append(x)
    if cur:
        launches.append((kid, cur))
# merge the attention merge-CTA records into their launch
rows = []
for kid, cs in launches:
    a = np.array(cs, dtype=rec.dtype)
    rows.append(dict(kind=L.TRACE_KIDS.get(int(kid), str(kid)), n=len(a), t0=int(a["t0"].min()),
                     w0=int(a["t1"].min()), w1=int(a["t1"].max()), t2=int(a["t2"].max()),
                     t2min=int(a["t2"].min())))
rows.sort(key=lambda d: d["t0"])
# the last decode pass: from the last add_ln whose predecessor is the final LN of the previous pass;
# simply take the launches after the last prefill-sized GEMM and split into passes at the LM head
gem = [i for i, d in enumerate(rows) if d["kind"] == "gemm"]
per_pass = 4 * cfg.n_layers + 1
start = gem[-per_pass]   # first GEMM (QKV layer 0) of the last pass
sel = [d for d in rows[start - 1:]]       # include LN1 of layer 0
T0 = sel[0]["t0"]
print(f"{'kind':>10} {'ctas':>5} {'entry':>9} {'wait_min':>9} {'wait_max':>9} {'exit_min':>9} {'exit':>9} {'span':>7}")
kinds_per_layer = None
for i, d in enumerate(sel):
    if i < 10 * nprint + 2 or i > len(sel) - 6:
        print(f"{d['kind']:>10} {d['n']:5d} {(d['t0']-T0)/1e3:9.2f} {(d['w0']-T0)/1e3:9.2f} {(d['w1']-T0)/1e3:9.2f} "
              f"{(d['t2min']-T0)/1e3:9.2f} {(d['t2']-T0)/1e3:9.2f} {(d['t2']-d['w1'])/1e3:7.2f}")
tot = (sel[-1]["t2"] - T0) / 1e3
print(f"pass (LN1 l0 entry .. last exit): {tot:.1f} us over {len(sel)} launches")
# critical-path attribution: time between consecutive launch exits
acc = {}
prev_end = sel[0]["t0"]
for d in sel:
    dt = max(0, d["t2"] - prev_end)
    acc[d["kind"]] = acc.get(d["kind"], 0) + dt
    prev_end = max(prev_end, d["t2"])
print("exit-to-exit attribution (us/pass):", {k: round(v / 1e3, 1) for k, v in acc.items()})
