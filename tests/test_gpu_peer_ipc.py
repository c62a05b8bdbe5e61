"""GPU, two processes on one GPU: ES_SCHED_PEER through real CUDA IPC.

Each process is one rank with its own CUDA context; the ranks exchange
es_peer_blob()s over torch.distributed (gloo) and map each other's
workspaces with cudaIpcOpenMemHandle -- the same code path as separate GPUs
over NVLink, except that the two contexts time-slice one device.  Three
global steps must give the oracle's bits on both ranks (D1)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, port, q, sched, options=0):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=2)
    try:
        import oracle
        from gpu_util import from_dev, to_dev
        from paper_conf_sc_lixyszrljlllq23_b200 import es
        from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator
        torch.cuda.set_device(0)
        N, mapping = 6, [0, 1, 1, 0, 1, 1]        # uneven: 2 and 4 local ESTs
        Ls, dts = [100003, 4096, 17], ["f32", "bf16", "f32"]
        agg = Aggregator(N, 2, rank, mapping, list(zip(Ls, dts)), transport=es.ES_TRANSPORT_NONE, sched=sched,
                         options=options)
        agg.peer_connect()
        ok = True
        for step in range(3):
            rng = np.random.default_rng(100 + step)         # same inputs in both processes
            xs = []
            for L, d in zip(Ls, dts):
                row = [(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
                xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
            loc = agg.local_ests
            devs = {k: [to_dev(xs[b][k]) for b in range(3)] for k in loc}
            for i, k in enumerate(loc):
                agg.stash_many(k, range(3), devs[k], es.ES_STASH_BORROW if i == len(loc) - 1 else es.ES_STASH_COPY)
            outs = [agg.new_out(b) for b in range(3)]
            agg.allreduce_many(range(3), outs)
            torch.cuda.synchronize()
            for b in range(3):
                got = from_dev(outs[b])
                want = oracle.reduce(xs[b], dts[b])
                ok &= bool(np.array_equal(got.view(np.uint8), want.view(np.uint8)))
        agg.sync()
        agg.close()
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("sched_name,opt_name", [("ES_SCHED_PEER", None), ("ES_SCHED_PEER_CHAIN", None),
                                                ("ES_SCHED_PEER", "ES_OPT_PEER_PUSH")])
def test_peer_schedule_two_processes_real_ipc(sched_name, opt_name):
    import sys
    sys.path.insert(0, ROOT)
    from paper_conf_sc_lixyszrljlllq23_b200 import es
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    options = getattr(es, opt_name) if opt_name else 0
    ps = [ctx.Process(target=_worker, args=(r, port, q, getattr(es, sched_name), options)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(timeout=300)
    for p in ps:
        if p.is_alive():
            p.kill()
    res = dict(q.get(timeout=5) for _ in range(2))
    assert res == {0: True, 1: True}
