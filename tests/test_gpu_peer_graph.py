"""GPU: the peer-memory schedules (PEER, PEER_CHAIN) replayed from CUDA
graphs, as bench.py runs every schedule.  The device barrier's epoch lives in
device memory, so replay i must wait for every peer's replay i: with new
inputs written in place before each replay, a barrier that passed early would
fold a peer's previous-step partials/results and miss the oracle's bits.
An eager step precedes the capture so the counters are not at zero
(eager and replayed barriers share one sequence)."""
import threading

import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads

from gpu_util import Aggregator, assert_bits_equal, code, from_dev, to_dev

pytestmark = pytest.mark.gpu


def _inputs(rng, N, Ls, dts):
    xs = []
    for L, d in zip(Ls, dts):
        row = [(rng.standard_normal(L) * 1e-2).astype(np.float32) for _ in range(N)]
        xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
    return xs


@pytest.mark.parametrize("sched,options", [(es.ES_SCHED_PEER, 0), (es.ES_SCHED_PEER_CHAIN, 0),
                                           (es.ES_SCHED_PEER_CHAIN, es.ES_OPT_PEER_ROUNDS),
                                           (es.ES_SCHED_PEER, es.ES_OPT_INCREMENTAL),
                                           (es.ES_SCHED_PEER_CHAIN, es.ES_OPT_INCREMENTAL),
                                           (es.ES_SCHED_PEER_AUTO, es.ES_OPT_INCREMENTAL | es.ES_OPT_PEER_ROUNDS)])
@pytest.mark.parametrize("G,N,kind", [(2, 8, "contiguous"), (4, 12, "random")])
def test_peer_schedules_under_graph_replay(sched, options, G, N, kind):
    Ls, dts = [120011, 4099, 33], ["f32", "bf16", "f32"]
    B = len(Ls)
    m = workloads.mapping(N, G, kind, seed=3) if kind == "random" else workloads.mapping(N, G, kind)
    rng = np.random.default_rng(40 + G + sched)
    xs = _inputs(rng, N, Ls, dts)
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, g, m, [(L, code(xs[b][0])) for b, L in enumerate(Ls)],
                       transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value, sched=sched, options=options)
            for g in range(G)]
    blobs = [a.peer_blob() for a in aggs]
    for a in aggs:
        a.peer_open(blobs)
    devs = [[to_dev(xs[b][k]) for b in range(B)] for k in range(N)]   # fixed addresses, rewritten per replay
    outs = [[a.new_out(b) for b in range(B)] for a in aggs]
    streams = [torch.cuda.Stream() for _ in range(G)]
    torch.cuda.synchronize()

    def step(g):
        a = aggs[g]
        for i, k in enumerate(a.local_ests):
            mode = es.ES_STASH_BORROW if i == len(a.local_ests) - 1 else es.ES_STASH_COPY
            if options & es.ES_OPT_INCREMENTAL:     # NEXT-1 at G > 1: fold at the stash
                a.stash_fold(k, range(B), devs[k], mode)
            else:
                a.stash_many(k, range(B), devs[k], mode)
        a.allreduce_many(range(B), outs[g])

    def on_threads(fn):
        errs = []

        def run(g):
            try:
                with torch.cuda.stream(streams[g]):
                    fn(g)
            except Exception as e:  # surfaced below
                errs.append(e)
        ts = [threading.Thread(target=run, args=(g,)) for g in range(G)]
        [t.start() for t in ts]
        [t.join(timeout=300) for t in ts]
        torch.cuda.synchronize()
        if errs:
            raise errs[0]

    def check(tag):
        for b in range(B):
            want = oracle.reduce(xs[b], dts[b])
            for g in range(G):
                assert_bits_equal(from_dev(outs[g][b]), want, f"{tag} rank {g} bucket {b}")

    on_threads(step)                                   # eager step: counters advance to a nonzero value
    check("eager")
    graphs = []
    for g in range(G):                                 # capture needs no peer to run: one rank at a time
        gr = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gr, stream=streams[g]):
            step(g)
        graphs.append(gr)
    torch.cuda.synchronize()
    for rep in range(4):
        xs = _inputs(rng, N, Ls, dts)
        for k in range(N):
            for b in range(B):
                devs[k][b].copy_(to_dev(xs[b][k]))
        for g in range(G):
            for o in outs[g]:
                o.zero_()
        torch.cuda.synchronize()
        on_threads(lambda g: graphs[g].replay())
        check(f"replay {rep}")
    on_threads(step)                                   # eager again after the replays
    check("eager after replays")
    for a in aggs:
        a.sync()
        a.close()
    es.es_loopback_destroy(world)


@pytest.mark.parametrize("options", [0, es.ES_OPT_PEER_ROUNDS])
def test_peer_chain_launch_structure(options):
    """The pipelined PEER_CHAIN step is [barrier] one k_fold_pipe per dtype
    [barrier] gather; ES_OPT_PEER_ROUNDS has a barrier between rounds."""
    N, G = 8, 2
    Ls, dts = [300007, 20011], ["f32", "bf16"]
    rng = np.random.default_rng(5)
    xs = _inputs(rng, N, Ls, dts)
    m = workloads.mapping(N, G, "contiguous")
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, g, m, [(L, code(xs[b][0])) for b, L in enumerate(Ls)],
                       transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value, sched=es.ES_SCHED_PEER_CHAIN,
                       options=options) for g in range(G)]
    blobs = [a.peer_blob() for a in aggs]
    for a in aggs:
        a.peer_open(blobs)
        a.profile(False)
        a.profile_reset()
    devs = [[to_dev(xs[b][k]) for b in range(2)] for k in range(N)]
    outs = [[a.new_out(b) for b in range(2)] for a in aggs]
    streams = [torch.cuda.Stream() for _ in range(G)]
    torch.cuda.synchronize()

    def run(g):
        with torch.cuda.stream(streams[g]):
            a = aggs[g]
            for i, k in enumerate(a.local_ests):
                a.stash_many(k, range(2), devs[k], es.ES_STASH_BORROW if i == len(a.local_ests) - 1 else es.ES_STASH_COPY)
            a.allreduce_many(range(2), outs[g])
    ts = [threading.Thread(target=run, args=(g,)) for g in range(G)]
    [t.start() for t in ts]
    [t.join(timeout=300) for t in ts]
    torch.cuda.synchronize()
    rounds = 3   # N=8 on G=2 contiguous: chunk c visits GPU(c+1), the other GPU, then GPU(c+1) again
    for g, a in enumerate(aggs):
        nb = a.profile_query(es.ES_KERNEL_BARRIER)[0]
        nf = a.profile_query(es.ES_KERNEL_FOLD)[0]
        if options == 0:
            assert (nb, nf) == (2, 2), (g, nb, nf)
        else:
            assert nb == rounds + 1 and nf >= 2 * (rounds - 1), (g, nb, nf)   # rank 1 has no round-2 folds
        for b in range(2):
            assert_bits_equal(from_dev(outs[g][b]), oracle.reduce(xs[b], dts[b]), f"rank {g} b {b}")
    for a in aggs:
        a.close()
    es.es_loopback_destroy(world)
