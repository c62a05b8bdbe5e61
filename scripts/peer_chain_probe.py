"""PEER_CHAIN on one GPU over the loopback transport: tile-pipelined
(k_fold_pipe, default) vs one launch per round with device barriers
(ES_OPT_PEER_ROUNDS).  Stashes are zero-copy (ES_STASH_INPLACE), so a step is
the allreduce.  All G ranks share this GPU, so both variants are bound
by the one HBM (no NVLink here); the comparison isolates what pipelining
removes -- the per-round barriers and the tail of each round.  Each rank's
step is captured in a CUDA graph and the G graphs
are replayed concurrently from G host threads; time = wall per step over the
replays.  Prints one JSON line per (config, G, variant).

  python scripts/peer_chain_probe.py [config] [G ...]
"""
import json
import os
import sys
import threading
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads  # noqa: E402
from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator  # noqa: E402


def run(name, G, options, iters=20):
    cfg = workloads.config(name)
    N, buckets = cfg["N"], cfg["buckets"]
    B = len(buckets)
    m = workloads.mapping(N, G, "contiguous")
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, g, m, buckets, transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value,
                       sched=es.ES_SCHED_PEER_CHAIN, options=options) for g in range(G)]
    blobs = [a.peer_blob() for a in aggs]
    for a in aggs:
        a.peer_open(blobs)
    # zero-copy stashes (ES_STASH_INPLACE): the gradients live in the slots, so a step is the allreduce
    grads = {}
    for a in aggs:
        for k in a.local_ests:
            grads[k] = [workloads.est_bucket(name, k, b, device="cuda", out=a.slot(k, b)) for b in range(B)]
    outs = [[a.new_out(b) for b in range(B)] for a in aggs]
    streams = [torch.cuda.Stream() for _ in range(G)]
    torch.cuda.synchronize()

    def step(g):
        a = aggs[g]
        for k in a.local_ests:
            a.stash_many(k, range(B), grads[k], es.ES_STASH_INPLACE)
        a.allreduce_many(range(B), outs[g])

    def on_threads(fn):
        def body(g):
            with torch.cuda.stream(streams[g]):
                fn(g)
        ts = [threading.Thread(target=body, args=(g,)) for g in range(G)]
        [t.start() for t in ts]
        [t.join() for t in ts]
        torch.cuda.synchronize()

    on_threads(step)                       # eager warm-up
    graphs = []
    for g in range(G):
        gr = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gr, stream=streams[g]):
            step(g)
        graphs.append(gr)
    torch.cuda.synchronize()
    for _ in range(3):
        on_threads(lambda g: graphs[g].replay())
    t0 = time.perf_counter()
    for _ in range(iters):
        on_threads(lambda g: graphs[g].replay())
    ms = (time.perf_counter() - t0) / iters * 1e3
    for a in aggs:
        a.sync()
        a.close()
    es.es_loopback_destroy(world)
    payload = workloads.payload_bytes(name)
    return {"probe": "peer_chain_loopback", "config": name, "N": N, "G": G,
            "variant": "rounds" if options else "pipelined", "ms_per_allreduce_step": round(ms, 4),
            "EST_GBps": round(payload / (ms / 1e3) / 1e9, 1)}


if __name__ == "__main__":
    name = sys.argv[1] if len(sys.argv) > 1 else "resnet50"
    Gs = [int(x) for x in sys.argv[2:]] or [2, 4]
    for G in Gs:
        variants = os.environ.get("PROBE_VARIANTS", "rounds,pipelined").split(",")
        for opt in [{"rounds": es.ES_OPT_PEER_ROUNDS, "pipelined": 0}[v] for v in variants]:
            print(json.dumps(run(name, G, opt)), flush=True)
