"""Dev: repeat the loopback TP=4 serial run with / without the fused all-reduce and
report per-rank outcomes (flakiness hunt)."""
import os, sys, time, threading
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from liger_inputs import make_trace
from liger_inputs.configs import ModelConfig
from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine as E
world = int(sys.argv[1]) if len(sys.argv) > 1 else 4
cfg = ModelConfig("mid2", 2, 1024, 8, 4096, 1024, 96, "relu")
trace = make_trace(3, float("inf"), seed=8, batch_sizes=(1, 3), prompt_range=(10, 40), n_decode=5, vocab=cfg.vocab)
for it in range(int(sys.argv[2]) if len(sys.argv) > 2 else 4):
    for flag in ("0", "1"):
        os.environ["LIGER_FUSED_AR"] = flag
        uid = E.loopback_id()
        out, err = [None] * world, [None] * world
        def rank_main(r):
            try:
                torch.cuda.set_device(0)
                eng = E(cfg, world=world, rank=r, nccl_uid=uid, mode="serial", max_batch=4, max_seq=48, max_new=8, seed=9)
                ids = [eng.submit(t["tokens"], t["batch"], t["seq_len"], t["n_decode"], 0.0) for t in trace]
                eng.drain()
                out[r] = ([eng.poll(i, want_tokens=True)[1] for i in ids], eng.stats())
                eng.close()
            except Exception as e:
                err[r] = repr(e)[:300]
        t0 = time.time()
        ths = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
        for t in ths: t.start()
        for t in ths: t.join(timeout=120)
        print(f"iter {it} fused={flag} {time.time() - t0:.1f}s errors={err} "
              f"comm={[o[1]['comm_kernels'] if o else None for o in out]}", flush=True)
        if any(err):
            sys.exit(1)
