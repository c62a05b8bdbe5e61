"""GPU: the NCCL transport's binding on a one-GPU box.  A world-size-1
ProcessGroupNCCL communicator is handed to es_init (G = 1): libes must
resolve the process's libnccl, accept the comm (size 1, rank 0) and reject a
communicator that does not match the config (include/es.h, es_transport).
The G > 1 NCCL data path itself runs in test_gpu_multi_nccl.py (>= 2 GPUs)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _worker(port, q):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        import oracle
        from gpu_util import from_dev, to_dev
        from paper_conf_sc_lixyszrljlllq23_b200 import es
        from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator, nccl_comm_ptr
        dist.all_reduce(torch.ones(1, device=dev))
        comm = nccl_comm_ptr()
        res = {"comm_nonzero": comm != 0}
        N, L = 3, 70001
        agg = Aggregator(N, 1, 0, [0] * N, [(L, "f32")], transport=es.ES_TRANSPORT_NCCL, comm=comm, device=dev)
        rng = np.random.default_rng(5)
        xs = [(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
        for k in range(N):
            agg.stash(k, 0, to_dev(xs[k]))
        out = agg.new_out(0)
        agg.allreduce(0, out)
        torch.cuda.synchronize()
        res["bits"] = bool(np.array_equal(from_dev(out).view(np.uint32), oracle.reduce(xs, "f32").view(np.uint32)))
        agg.close()
        try:                                       # rank 1 of a size-1 comm: must be refused
            Aggregator(2, 2, 1, [0, 1], [(L, "f32")], transport=es.ES_TRANSPORT_NCCL, comm=comm, device=dev)
            res["mismatch"] = "accepted"
        except es.EsError as e:
            res["mismatch"] = e.status == es.ES_ENCCL
        q.put(res)
    finally:
        dist.destroy_process_group()


def test_nccl_comm_binding_single_gpu():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_worker, args=(port, q))
    p.start()
    p.join(timeout=240)
    if p.is_alive():
        p.kill()
    assert q.get(timeout=5) == {"comm_nonzero": True, "bits": True, "mismatch": True}
