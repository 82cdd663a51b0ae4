"""Target for ncu launch lists: one OPT-13B batch (prefill + decode) through the
engine, no duration profiling.  Usage: python tools/profile_run.py [b] [s] [n_new]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from liger_inputs import get_config
from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
b, s, n = (int(a) for a in (sys.argv[1:4] if len(sys.argv) >= 4 else (4, 256, 8)))
cfg = get_config(os.environ.get("CFG", "opt-13b"))
eng = LigerEngine(cfg, mode="interleaved", max_batch=8, max_seq=512, max_new=32, seed=0)
toks = np.random.default_rng(0).integers(0, cfg.vocab, size=b * s).astype(np.int32)
for _ in range(2):
    eng.submit(toks, b, s, n, 0.0)
    eng.drain()
torch.cuda.synchronize()
print("done", eng.stats())
