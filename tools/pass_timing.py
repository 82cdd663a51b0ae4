"""Dev: device time of a decode pass through the engine (OPT-13B TP=1), from the
difference of batches with n_new = 32 and n_new = 1 (31 decode passes)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from liger_inputs import get_config
from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
cfg = get_config("opt-13b")
eng = LigerEngine(cfg, mode="serial", max_batch=8, max_seq=512, max_new=32, seed=0)
b, s = int(sys.argv[1]) if len(sys.argv) > 1 else 8, 256
toks = torch.from_numpy(np.random.default_rng(0).integers(0, cfg.vocab, size=b * s).astype(np.int32)).cuda()
def run(n_new, reps=3):
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        eng.submit(None, b, s, n_new, 0.0, device_tokens=toks)
        eng.drain()
        e.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(e))
    return min(ts)
run(2)
t1, t32 = run(1), run(32)
print(f"b={b} s={s}: prefill-only batch {t1:.2f} ms; 31 decode passes {t32 - t1:.2f} ms -> {(t32 - t1) / 31 * 1e3:.0f} us/pass "
      f"(PDL {'off' if os.environ.get('LIGER_NO_PDL') else 'on'})")
