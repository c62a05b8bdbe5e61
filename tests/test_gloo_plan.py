"""CPU, world_size 2 (gloo): two real processes each execute their own rank's
plan (exported from libes through the C ABI) and exchange the planned
messages with torch.distributed point-to-point -- the multi-process shape of
the NCCL path, on CPU.  Both ranks must end with the oracle's bits."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class GlooTransport:
    """NCCL-like matching: the n-th message from a to b carries tag n."""

    def __init__(self):
        self.sent = {}
        self.recvd = {}

    def group(self, ex, body):
        reqs, pend = [], []
        for f in body:
            peer = int(f[3])
            if int(f[0]) == 2:   # ES_OP_SEND
                data = ex._payload(f)
                t = torch.from_numpy(data.view(np.int16) if data.dtype == np.uint16 else data)
                tag = self.sent.get(peer, 0)
                self.sent[peer] = tag + 1
                reqs.append(dist.isend(t, dst=peer, tag=tag))
            else:
                n = int(f[2]) - int(f[1])
                kind = int(f[4])
                bdt = ex.buckets[ex.b][1]
                if kind == 3 or bdt == "f32":                  # ES_BUF_PART is fp32
                    buf = torch.empty(n, dtype=torch.float32)
                else:
                    buf = torch.empty(n, dtype=torch.int16)
                tag = self.recvd.get(peer, 0)
                self.recvd[peer] = tag + 1
                reqs.append(dist.irecv(buf, src=peer, tag=tag))
                pend.append((f, buf))
        for r in reqs:
            r.wait()
        for f, buf in pend:
            a = buf.numpy()
            ex._deliver(f, a.view(np.uint16) if a.dtype == np.int16 else a)
        return True


def _worker(rank, world, port, N, mapping, sched, q):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from plan_sim import RankExec
        rng = np.random.default_rng(77)
        Ls, dts = [4099, 1000, 17], ["f32", "bf16", "f32"]
        xs = []
        for L, d in zip(Ls, dts):
            row = [(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
            xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
        ex = RankExec(N, world, rank, mapping, list(zip(Ls, dts)), xs, sched=sched)
        tp = GlooTransport()
        while not ex.done():
            ex.run(tp)
        ok = all(np.array_equal(ex.out[b].view(np.uint32 if d == "f32" else np.uint16),
                                oracle.reduce(xs[b], d).view(np.uint32 if d == "f32" else np.uint16))
                 for b, d in enumerate(dts))
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("N,mapping,sched", [(4, [0, 0, 1, 1], 1), (4, [0, 0, 1, 1], 2), (5, [1, 0, 0, 1, 0], 2),
                                             (5, [1, 0, 0, 1, 0], 1), (12, [k % 2 for k in range(12)], 0)])
def test_two_process_gloo_plan(N, mapping, sched):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, N, mapping, sched, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=180)
    res = dict(q.get(timeout=10) for _ in range(2))
    assert all(p.exitcode == 0 for p in procs)
    assert res == {0: True, 1: True}
