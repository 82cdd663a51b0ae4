"""The CUDA-IPC one-shot all-reduce transport across two PROCESSES (it had only
run inside one process).  Two processes on the one GPU of this box each allocate a
peer-visible staging region (liger_ipc_region_create), exchange the 64-byte IPC handles over
a gloo process group, map the peer's region (liger_ipc_region_open) and run
liger_op_oneshot_allreduce -- stage, system-scope epoch flag, rank-ordered fp32 sum -- on
seeded bf16 partials, element-wise against the oracle's sum (bit-exact at t = 2: the sum of
two bf16 values is exact in fp32 and rounds once).  Both ranks must end with the same bits.

The two processes share one GPU, where kernels that wait on each other are not guaranteed
to be co-scheduled (B200_PROFILING.md: such process pairs raised Xid 109).  Each call
therefore runs in two phases: both ranks stage + publish (LIGER_AR_PHASE_STAGE) and
synchronise, a gloo barrier, then both wait + sum (LIGER_AR_PHASE_REDUCE) -- whose flag
waits are already satisfied -- so the peer loads, flags and IPC mappings are exercised
across processes without any kernel spinning on another process's kernel."""
import os

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu

CAP = 1 << 20


def _rank(r, port, q):
    import torch.distributed as dist
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=r, world_size=2)
        torch.cuda.set_device(0)
        from liger_inputs import c0_values
        from paper_conf_ppopp_duwjchcl24_b200 import liger as L
        region, handle = L.ipc_region_create(CAP)
        hs = [None, None]
        dist.all_gather_object(hs, handle)
        regions = [region if k == r else L.ipc_region_open(hs[k]) for k in range(2)]
        out = []
        for e, n in enumerate((8 * 5120, 16 * 1024, 256), start=1):
            x = c0_values(5, 200 + r, np.arange(n, dtype=np.uint64) + 1000 * e, -3)
            buf = torch.from_numpy(x.astype(np.float32)).cuda().bfloat16()
            L.oneshot_allreduce(buf, regions, r, CAP, e, phases=L.AR_PHASE_STAGE)
            torch.cuda.synchronize()
            dist.barrier()
            L.oneshot_allreduce(buf, regions, r, CAP, e, phases=L.AR_PHASE_REDUCE)
            torch.cuda.synchronize()
            dist.barrier()
            out.append(buf.view(torch.int16).cpu().numpy().tobytes())
        dist.barrier()
        for k in range(2):
            if k != r:
                L.lib().liger_ipc_region_close(regions[k])
        dist.barrier()
        L.lib().liger_ipc_region_free(region)
        q.put((r, out, None))
        dist.destroy_process_group()
    except Exception as ex:   # reported to the parent
        q.put((r, None, repr(ex)))


def test_oneshot_allreduce_across_two_processes():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    from liger_inputs import c0_values, bf16_rne
    import bench
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = bench._free_port()
    ps = [ctx.Process(target=_rank, args=(r, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = dict((r, (o, e)) for r, o, e in (q.get(timeout=240) for _ in range(2)))
    for p in ps:
        p.join(timeout=60)
    assert res[0][1] is None and res[1][1] is None, (res[0][1], res[1][1])
    assert res[0][0] == res[1][0]   # both ranks hold the same bits
    for e, n in enumerate((8 * 5120, 16 * 1024, 256), start=1):
        parts = [c0_values(5, 200 + r, np.arange(n, dtype=np.uint64) + 1000 * e, -3).astype(np.float64)
                 for r in range(2)]
        want = bf16_rne((parts[0] + parts[1]).astype(np.float32))
        got = np.frombuffer(res[0][0][e - 1], dtype=np.int16)
        assert np.array_equal(got, (want.view(np.uint32) >> 16).astype(np.uint16).view(np.int16))
