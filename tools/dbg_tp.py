import sys, threading, numpy as np, torch
sys.path.insert(0, '/root/repo'); sys.path.insert(0, '/root/repo/tests')
from liger_inputs import get_config, make_trace
from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine as E
cfg = get_config("tiny")
trace = make_trace(5, float("inf"), seed=11, batch_sizes=(1, 2, 3), prompt_range=(8, 40), n_decode=6, vocab=cfg.vocab)
print([(t["batch"], t["seq_len"]) for t in trace])
for world, mode in ((1, "serial"), (2, "serial"), (2, "interleaved")):
    uid = E.loopback_id() if world > 1 else None
    res = [None] * world
    def rank_main(r):
        eng = E(cfg, world=world, rank=r, nccl_uid=uid, mode=mode, max_batch=4, max_seq=64, max_new=8, seed=3)
        ids = [eng.submit(t["tokens"], t["batch"], t["seq_len"], t["n_decode"], 0.0) for t in trace]
        eng.drain()
        res[r] = ([eng.poll(i) is not None for i in ids], eng.stats())
        eng.close()
    ths = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    [t.start() for t in ths]; [t.join() for t in ths]
    print(world, mode, res)
