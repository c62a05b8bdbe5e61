"""NEXT-3 (iii): how close is the canonical order (R1/R2) to a real NCCL ring?

Needs N = G GPUs (one EST per GPU, the paper's DDP case).  Run with

  NCCL_ALGO=Ring NCCL_PROTO=Simple NCCL_MAX_NCHANNELS=1 \\
  torchrun --nproc-per-node 8 --master-addr 127.0.0.1 scripts/nccl_ring_probe.py

Every rank contributes its seeded bucket; rank 0 compares, word by word,
(a) es_allreduce (canonical order, bit-exact with the oracle) with
(b) torch.distributed.all_reduce(SUM) over NCCL followed by the same fl32(1/N)
post-scale, for several bucket sizes, and prints one JSON line with the
fraction of identical words.  Reading R2 claims (a) is "the order an N-worker
ring uses"; NCCL's own chunking (chunkSize, slices, channels) and its ring
order decide whether (b) agrees.  The paper does not pin this (DESIGN.md §3,
"parity unpinned"); this probe measures it.
"""
import json
import os
import sys

import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sc_lixyszrljlllq23_b200 import es  # noqa: E402
from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator, nccl_comm_ptr  # noqa: E402


def main():
    rank, G = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", rank)))
    dev = torch.device("cuda", torch.cuda.current_device())
    dist.init_process_group("nccl", device_id=dev)
    dist.all_reduce(torch.ones(1, device=dev))
    N = G
    r = torch.tensor(1.0, dtype=torch.float32) / torch.tensor(float(N), dtype=torch.float32)
    res = {}
    for L in (1 << 12, 1 << 16, 1 << 20, 25 << 20 >> 2):
        agg = Aggregator(N, G, rank, list(range(G)), [(L, "f32")], transport=es.ES_TRANSPORT_NCCL,
                         comm=nccl_comm_ptr(), sched=es.ES_SCHED_DIRECT, device=dev)
        g = torch.Generator(device=dev).manual_seed(1000 + rank)
        x = torch.randn(L, generator=g, device=dev) * 1e-3
        agg.stash(rank, 0, x, es.ES_STASH_COPY)
        canon = agg.new_out(0)
        agg.allreduce(0, canon)
        ring = x.clone()
        dist.all_reduce(ring)                    # NCCL's own order
        ring = ring * r.item()
        torch.cuda.synchronize()
        same = (canon.view(torch.int32) == ring.view(torch.int32)).float().mean().item()
        res[str(L)] = round(same, 6)
        agg.close()
    if rank == 0:
        print(json.dumps({"probe": "nccl_ring_vs_canonical", "N": N, "env": {k: os.environ.get(k) for k in
                          ("NCCL_ALGO", "NCCL_PROTO", "NCCL_MAX_NCHANNELS")}, "identical_word_fraction": res}))
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
