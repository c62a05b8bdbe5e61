"""Probe: can two NCCL ranks share one GPU (two processes, same device)?"""
import os
import sys

import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def w(rank, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    try:
        dist.init_process_group("nccl", rank=rank, world_size=2, device_id=torch.device("cuda", 0))
        t = torch.ones(4, device="cuda") * (rank + 1)
        dist.all_reduce(t)
        torch.cuda.synchronize()
        q.put((rank, float(t[0])))
        dist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e)[:300]))


if __name__ == "__main__":
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=w, args=(r, 29533, q)) for r in range(2)]
    [p.start() for p in ps]
    [p.join(120) for p in ps]
    for p in ps:
        if p.is_alive():
            p.kill()
    out = []
    while not q.empty():
        out.append(q.get())
    print("probe:", out)
    sys.exit(0)
