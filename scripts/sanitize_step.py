"""Small end-to-end workload for compute-sanitizer (memcheck / racecheck /
initcheck / synccheck): every kernel and API path of libes once, on tiny
ragged buckets, with bit-exact checks against the oracle.

  compute-sanitizer --tool memcheck python scripts/sanitize_step.py
"""
import os
import sys
import threading

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import oracle  # noqa: E402
from gpu_util import assert_bits_equal, from_dev, to_dev  # noqa: E402
from paper_conf_sc_lixyszrljlllq23_b200 import es  # noqa: E402
from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator  # noqa: E402


def data(rng, N, Ls, dts):
    xs = []
    for L, d in zip(Ls, dts):
        row = [(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
        xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
    return xs


def g1(rng, options=0):
    N, Ls, dts = 5, [1001, 17, 64, 3], ["f32", "bf16", "f32", "bf16"]
    sizes = [16, 4096, 37]
    agg = Aggregator(N, 1, 0, [0] * N, list(zip(Ls, dts)), state_nbytes=sizes, options=options)
    live = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
    agg.register_state(live)
    for k in range(N):
        for i, n in enumerate(sizes):
            agg.init_state(k, i, bytes(rng.integers(0, 256, n, dtype=np.uint8)))
    xs = data(rng, N, Ls, dts)
    devs = [[to_dev(xs[b][k]) for b in range(len(Ls))] for k in range(N)]
    outs = [agg.new_out(b) for b in range(len(Ls))]
    agg.switch(0)
    for k in range(N):
        if k == N - 1:
            agg.stash_many(k, range(len(Ls)), devs[k], es.ES_STASH_BORROW)
        else:
            agg.stash_and_switch(k, range(len(Ls)), devs[k], k + 1)
    agg.allreduce_many(range(len(Ls)), outs)
    y, m = agg.dropout(torch.ones(1001, device="cuda"), 0.3, with_mask=True)
    torch.cuda.synchronize()
    for b, d in enumerate(dts):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], d), f"g1 b={b}")
    blob = agg.export_context(2)
    agg.import_context(2, blob)
    agg.close()
    inc = Aggregator(N, 1, 0, [0] * N, list(zip(Ls, dts)), options=options | es.ES_OPT_INCREMENTAL)
    for k in range(N):
        inc.stash_fold(k, range(len(Ls)), devs[k])
    inc.allreduce_many(range(len(Ls)), outs)
    torch.cuda.synchronize()
    for b, d in enumerate(dts):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], d), f"incremental b={b}")
    inc.close()


def multi(rng, sched, options=0, big=False):
    N, G, m = 6, 3, [0, 1, 2, 2, 0, 1]
    Ls, dts = [1003, 40, 9], ["f32", "bf16", "f32"]
    if big:   # chunks above 2^20 elements: the tile-pipelined CHAIN cuts them into W = 2 tiles
        N, G, m = 4, 2, [0, 0, 1, 1]
        Ls, dts = [4 * (1 << 20) + 4 * 4096 + 3, 40], ["f32", "bf16"]
    xs = data(rng, N, Ls, dts)
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, g, m, list(zip(Ls, dts)), transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value,
                       sched=sched, options=options) for g in range(G)]
    if sched in es.PEER_SCHEDS:
        blobs = [a.peer_blob() for a in aggs]
        for a in aggs:
            a.peer_open(blobs)
    devs = [[to_dev(xs[b][k]) for b in range(len(Ls))] for k in range(N)]
    outs = [[a.new_out(b) for b in range(len(Ls))] for a in aggs]
    streams = [torch.cuda.Stream() for _ in range(G)]
    torch.cuda.synchronize()
    errs = []

    def run(g):
        try:
            with torch.cuda.stream(streams[g]):
                loc = aggs[g].local_ests
                for i, k in enumerate(loc):
                    mode = es.ES_STASH_BORROW if i == len(loc) - 1 else es.ES_STASH_COPY
                    if options & es.ES_OPT_INCREMENTAL:     # NEXT-1 at G > 1
                        aggs[g].stash_fold(k, range(len(Ls)), devs[k], mode)
                    else:
                        aggs[g].stash_many(k, range(len(Ls)), devs[k], mode)
                aggs[g].allreduce_many(range(len(Ls)), outs[g])
        except Exception as e:
            errs.append(e)
    ts = [threading.Thread(target=run, args=(g,)) for g in range(G)]
    [t.start() for t in ts]
    [t.join() for t in ts]
    torch.cuda.synchronize()
    if errs:
        raise errs[0]
    for g in range(G):
        for b, d in enumerate(dts):
            assert_bits_equal(from_dev(outs[g][b]), oracle.reduce(xs[b], d), f"sched {sched} rank {g} b={b}")
    for a in aggs:
        a.close()
    es.es_loopback_destroy(world)


SCHEDS = {"direct": (es.ES_SCHED_DIRECT, 0), "chain": (es.ES_SCHED_CHAIN, 0), "peer": (es.ES_SCHED_PEER, 0),
          "peer_chain": (es.ES_SCHED_PEER_CHAIN, 0),
          "peer_chain_rounds": (es.ES_SCHED_PEER_CHAIN, es.ES_OPT_PEER_ROUNDS),
          "peer_push": (es.ES_SCHED_PEER, es.ES_OPT_PEER_PUSH),
          "chain_rounds": (es.ES_SCHED_CHAIN, es.ES_OPT_PEER_ROUNDS),
          "chain_tiles": (es.ES_SCHED_CHAIN, 0, True),
          "direct_inc": (es.ES_SCHED_DIRECT, es.ES_OPT_INCREMENTAL),
          "chain_inc": (es.ES_SCHED_CHAIN, es.ES_OPT_INCREMENTAL),
          "peer_inc": (es.ES_SCHED_PEER, es.ES_OPT_INCREMENTAL),
          "peer_chain_rounds_inc": (es.ES_SCHED_PEER_CHAIN, es.ES_OPT_PEER_ROUNDS | es.ES_OPT_INCREMENTAL)}

if __name__ == "__main__":
    # argv: which parts to run (default: all): g1 g1_bg and the SCHEDS keys
    parts = sys.argv[1:] or ["g1", "g1_bg"] + list(SCHEDS)
    rng = np.random.default_rng(0)
    for part in parts:
        if part == "g1":
            g1(rng)
        elif part == "g1_bg":
            g1(rng, es.ES_OPT_STASH_BACKGROUND)    # TMA-ring stash (k_copy_tma<4, 4096>) and capped grids
        else:
            multi(rng, *SCHEDS[part])
        print("part ok:", part, flush=True)
    print("sanitize_step ok")
