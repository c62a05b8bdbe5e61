"""Subprocess body of tests/test_gpu_knobs.py: run the hot path under whatever
libes environment knobs the parent set (ES_NO_PDL, ES_STASH_EARLY, ES_FOLD_TMA,
ES_BARRIER_TIMEOUT_S) and compare every output with the oracle bit for bit.

  python tests/knob_probe.py parity     -> prints KNOB_PROBE_OK
  python tests/knob_probe.py stuck      -> one peer rank never arrives: the
                                           barrier must trap (ES_ECUDA at sync)
"""
import os
import sys
import threading

import numpy as np
import torch

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(HERE))
sys.path.insert(0, HERE)

import oracle  # noqa: E402
from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads  # noqa: E402
from gpu_util import Aggregator, assert_bits_equal, code, from_dev, to_dev  # noqa: E402

Ls, DTS = [300007, 4099, 1 << 18, 17], ["f32", "bf16", "f32", "f32"]


def inputs(N, seed):
    rng = np.random.default_rng(seed)
    xs = []
    for L, d in zip(Ls, DTS):
        row = [(rng.standard_normal(L) * 1e-2).astype(np.float32) for _ in range(N)]
        xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
    return xs


def check(outs, xs, tag):
    for b in range(len(Ls)):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], DTS[b]), f"{tag} bucket {b}")


def g1_graph_step():
    """The bench's fused step (switch-in, stash+switch per EST, BORROW last,
    one batched allreduce) captured in a CUDA graph: consecutive stashes start
    early unless ES_STASH_EARLY=0; PDL unless ES_NO_PDL=1; TMA fold if ES_FOLD_TMA=1."""
    N, B = 8, len(Ls)
    xs = inputs(N, 1)
    snb = workloads.state_nbytes()
    agg = Aggregator(N, 1, 0, [0] * N, [(L, d) for L, d in zip(Ls, DTS)], state_nbytes=snb)
    live = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in snb]
    agg.register_state(live)
    for k in range(N):
        for i, blob in enumerate(workloads.est_state("tiny", k)):
            agg.init_state(k, i, blob)
    devs = [[to_dev(xs[b][k]) for b in range(B)] for k in range(N)]
    outs = [agg.new_out(b) for b in range(B)]

    def step():
        agg.switch(0)
        for k in range(N):
            if k == N - 1:
                agg.stash_many(k, range(B), devs[k], es.ES_STASH_BORROW)
            else:
                agg.stash_and_switch(k, range(B), devs[k], k + 1, es.ES_STASH_COPY)
        agg.allreduce_many(range(B), outs)

    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        step()
    torch.cuda.synchronize()
    check(outs, xs, "eager")
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        step()
    xs2 = inputs(N, 2)                                    # new inputs at the same addresses
    for k in range(N):
        for b in range(B):
            devs[k][b].copy_(to_dev(xs2[b][k]))
    for o in outs:
        o.zero_()
    with torch.cuda.stream(s):
        g.replay()
    torch.cuda.synchronize()
    agg.sync()
    check(outs, xs2, "graph replay")
    agg.close()


def loopback_peer(sched, G=2, N=8):
    xs = inputs(N, 3 + sched)
    B = len(Ls)
    m = workloads.mapping(N, G, "contiguous")
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, g, m, [(L, d) for L, d in zip(Ls, DTS)], transport=es.ES_TRANSPORT_LOOPBACK,
                       comm=world.value, sched=sched) for g in range(G)]
    blobs = [a.peer_blob() for a in aggs]
    for a in aggs:
        a.peer_open(blobs)
    devs = [[to_dev(xs[b][k]) for b in range(B)] for k in range(N)]
    outs = [[a.new_out(b) for b in range(B)] for a in aggs]
    streams = [torch.cuda.Stream() for _ in range(G)]
    torch.cuda.synchronize()
    errs = []

    def run(g):
        try:
            a = aggs[g]
            with torch.cuda.stream(streams[g]):
                for step in range(2):
                    for i, k in enumerate(a.local_ests):
                        a.stash_many(k, range(B), devs[k],
                                     es.ES_STASH_BORROW if i == len(a.local_ests) - 1 else es.ES_STASH_COPY)
                    a.allreduce_many(range(B), outs[g])
        except Exception as e:  # surfaced below
            errs.append(e)
    ts = [threading.Thread(target=run, args=(g,)) for g in range(G)]
    [t.start() for t in ts]
    [t.join(timeout=120) for t in ts]
    torch.cuda.synchronize()
    if errs:
        raise errs[0]
    for g in range(G):
        check(outs[g], xs, f"loopback sched {sched} rank {g}")
    for a in aggs:
        a.sync()
        a.close()
    es.es_loopback_destroy(world)


def stuck():
    """Rank 0 of a PEER pair enters the step's barrier; rank 1 never does."""
    N, G = 4, 2
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, g, [0, 0, 1, 1], [(4096, "f32")], transport=es.ES_TRANSPORT_LOOPBACK,
                       comm=world.value, sched=es.ES_SCHED_PEER) for g in range(G)]
    blobs = [a.peer_blob() for a in aggs]
    for a in aggs:
        a.peer_open(blobs)
    x = torch.ones(4096, device="cuda")
    out = aggs[0].new_out(0)
    for k in aggs[0].local_ests:
        aggs[0].stash(k, 0, x, es.ES_STASH_COPY)
    aggs[0].allreduce(0, out)
    try:
        aggs[0].sync()
    except es.EsError as e:
        print("STUCK_TRAPPED", e, flush=True)
        os._exit(0)
    print("STUCK_NOT_TRAPPED", flush=True)
    os._exit(1)


if __name__ == "__main__":
    torch.cuda.set_device(0)
    if sys.argv[1] == "stuck":
        stuck()
    g1_graph_step()
    loopback_peer(es.ES_SCHED_PEER)
    loopback_peer(es.ES_SCHED_PEER_CHAIN)
    print("KNOB_PROBE_OK", flush=True)
