"""Target for `ncu --set full`: OPT-13B TP = 1 served through the engine (b = 8, prompt 256,
2 generated tokens); the decode pass runs the folded-LN / residual-epilogue GEMMs
(gemm_tc_kernel<1>) -- capture the first four launches of that instantiation (layer 0's QKV,
out-proj, FC1, FC2 of the decode pass)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from liger_inputs import get_config
from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
cfg = get_config("opt-13b")
eng = LigerEngine(cfg, mode="serial", max_batch=8, max_seq=512, max_new=32, seed=0)
toks = torch.from_numpy(np.random.default_rng(0).integers(0, cfg.vocab, size=8 * 256).astype(np.int32)).cuda()
eng.submit(None, 8, 256, 2, 0.0, device_tokens=toks)
eng.drain()
torch.cuda.synchronize()
eng.close()
