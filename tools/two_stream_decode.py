"""Dev: aggregate decode weight-stream rate of the t = 1 two-stream schedule.

    python tools/two_stream_decode.py [b] [prompt] [mode]

Times (CUDA events, OPT-13B TP = 1) k equal batches served together, with 32 and with 1
generated tokens; (T32 - T1) / (k * 31) is the time per decode pass of one batch while k
batches decode concurrently; bytes = weights + KV read per pass."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from liger_inputs import get_config
from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine


def main():
    b = int(sys.argv[1]) if len(sys.argv) > 1 else 8
    s = int(sys.argv[2]) if len(sys.argv) > 2 else 256
    mode = sys.argv[3] if len(sys.argv) > 3 else "interleaved"
    cfg = get_config("opt-13b")
    eng = LigerEngine(cfg, mode=mode, max_batch=8, max_seq=512, max_new=32, max_inflight=2, seed=0)
    toks = np.random.default_rng(0).integers(0, cfg.vocab, size=b * s).astype(np.int32)

    def run(k, n):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        for _ in range(k):
            eng.submit(toks, b, s, n, 0.0)
        eng.drain()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) * 1e3

    run(2, 4)
    wbytes = 12 * cfg.hidden * cfg.hidden * 2 * cfg.n_layers   # 4h^2 + 2*4h^2 per layer, bf16
    kv = lambda pos: b * cfg.hidden * 2 * 2 * pos * cfg.n_layers
    for k in (1, 2):
        t32 = min(run(k, 32) for _ in range(3))
        t1 = min(run(k, 1) for _ in range(3))
        per = (t32 - t1) / (k * 31)
        byt = wbytes + kv(s + 16)
        print(f"{mode} k={k} b={b} s={s}: T32 {t32:.0f} us, T1 {t1:.0f} us, per-batch decode pass {per:.1f} us, "
              f"aggregate {byt / per / 1e3:.0f} GB/s")
    eng.close()


if __name__ == "__main__":
    main()
