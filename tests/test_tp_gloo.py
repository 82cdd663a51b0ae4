"""World-size-2 CPU (gloo) coverage of the N>1 data path (task ⑤).

Each rank holds only its Megatron shard and the two per-layer
all-reduces are real `torch.distributed` collectives; the result must equal the
unsharded oracle layer.  The chunked all-reduce (decomposition into F pieces,
P:254) must give the same values as the whole one.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from liger_inputs import get_config, layer_activation


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from oracle import model as om
    cfg = get_config("tiny")
    w = om.layer_weights(cfg, 0, 0)
    mine = om.shard_layer(cfg, w, world, rank)
    x = layer_activation(cfg, 0, 0, 2 * 5).astype(np.float64).reshape(2, 5, cfg.hidden)

    def ar(part, chunks=1):
        t = torch.from_numpy(np.ascontiguousarray(part)).reshape(-1)
        n = t.numel()
        for c in range(chunks):
            sl = t[c * n // chunks:(c + 1) * n // chunks]
            dist.all_reduce(sl)   # views share storage: reduced in place
        return t.reshape(part.shape).numpy()

    sub = om._LocalCfg(cfg, world)
    o, _, _ = om.attention_block(sub, mine, x)
    x1 = x + ar(o @ mine["w_o"], chunks=8) + w["b_o"]
    y2 = om.layer_norm(x1, w["ln2_g"], w["ln2_b"], cfg.ln_eps)
    p2 = om.activation(cfg)(y2 @ mine["w_1"] + mine["b_1"]) @ mine["w_2"]
    x2 = x1 + ar(p2) + w["b_2"]
    ref, _, _ = om.decoder_layer(cfg, w, x)
    out_q.put((rank, float(np.max(np.abs(x2 - ref)))))
    dist.destroy_process_group()


def test_tp2_gloo_layer_equals_unsharded():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert max(res.values()) < 1e-12
