"""Multi-GPU (runs only when >= 2 GPUs are visible; skipped on the 1-GPU
boxes of this build): the real NCCL transport and the real cross-GPU CUDA
IPC path, one process per GPU as bench.py runs them.  For G in {2, 4, 8}
(as many as are visible) and every schedule, every rank must hold the
oracle's bits for the same N = 8 ESTs (D1)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NGPU = torch.cuda.device_count() if torch.cuda.is_available() else 0


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, G, port, sched_name, q, options=0):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(rank)
    dev = torch.device("cuda", rank)
    dist.init_process_group("nccl", rank=rank, world_size=G, device_id=dev)
    try:
        import oracle
        from gpu_util import from_dev, to_dev
        from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads
        from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator, nccl_comm_ptr
        t = torch.ones(1, device=dev)
        dist.all_reduce(t)
        sched = getattr(es, sched_name)
        N = 8
        m = workloads.mapping(N, G, "contiguous")
        Ls, dts = [200003, 4099, 17], ["f32", "bf16", "f32"]
        agg = Aggregator(N, G, rank, m, list(zip(Ls, dts)), transport=es.ES_TRANSPORT_NCCL, comm=nccl_comm_ptr(),
                         sched=sched, device=dev, options=options)
        if sched in es.PEER_SCHEDS:
            agg.peer_connect()
        ok = True
        for step in range(2):
            rng = np.random.default_rng(10 + step)
            xs = []
            for L, d in zip(Ls, dts):
                row = [(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
                xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
            devs = {k: [to_dev(xs[b][k]).to(dev) for b in range(3)] for k in agg.local_ests}
            for i, k in enumerate(agg.local_ests):
                mode = es.ES_STASH_BORROW if i == len(agg.local_ests) - 1 else es.ES_STASH_COPY
                if options & es.ES_OPT_INCREMENTAL:          # NEXT-1 across real GPUs
                    agg.stash_fold(k, range(3), devs[k], mode)
                else:
                    agg.stash_many(k, range(3), devs[k], mode)
            outs = [agg.new_out(b) for b in range(3)]
            agg.allreduce_many(range(3), outs)
            torch.cuda.synchronize()
            for b in range(3):
                ok &= bool(np.array_equal(from_dev(outs[b]).view(np.uint8), oracle.reduce(xs[b], dts[b]).view(np.uint8)))
        agg.sync()
        agg.close()
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.skipif(NGPU < 2, reason="needs >= 2 GPUs (this build's boxes have one)")
@pytest.mark.parametrize("G", [g for g in (2, 4, 8) if g <= NGPU] or [2])
@pytest.mark.parametrize("sched_name", ["ES_SCHED_DIRECT", "ES_SCHED_CHAIN", "ES_SCHED_AUTO", "ES_SCHED_PEER",
                                        "ES_SCHED_PEER_CHAIN"])
@pytest.mark.parametrize("options", [0, 1, 2], ids=["default", "incremental", "rounds"])
def test_nccl_and_peer_paths_on_real_gpus(G, sched_name, options):
    """options: 0 (tile-pipelined CHAIN / PEER_CHAIN), 1 = ES_OPT_INCREMENTAL (NEXT-1),
    2 = ES_OPT_PEER_ROUNDS (the round executors)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, G, port, sched_name, q, options)) for r in range(G)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(timeout=300)
    for p in ps:
        if p.is_alive():
            p.kill()
    res = dict(q.get(timeout=5) for _ in range(G))
    assert res == {r: True for r in range(G)}
