"""Helpers for the -m gpu parity tests: drive the CUDA path through the C ABI
(via the thin binding) on seeded host inputs, and compare with the oracle.
The inputs are NumPy arrays (float32, or uint16 bf16 bit patterns) made by
the tests or by workloads.py; nothing here computes the method."""
import threading

import numpy as np
import torch

from paper_conf_sc_lixyszrljlllq23_b200 import es
from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator


def to_dev(x):
    x = np.ascontiguousarray(x)
    if x.dtype == np.float32:
        return torch.from_numpy(x).cuda()
    assert x.dtype == np.uint16
    return torch.from_numpy(x.view(np.int16)).cuda().view(torch.bfloat16)


def from_dev(t):
    t = t.detach().cpu()
    if t.dtype == torch.float32:
        return t.numpy()
    return t.view(torch.int16).numpy().view(np.uint16)


def code(x):
    return "f32" if np.asarray(x).dtype == np.float32 else "bf16"


def bits(a):
    a = np.asarray(a)
    return a.view(np.uint32) if a.dtype == np.float32 else a.view(np.uint16)


def assert_bits_equal(got, want, what=""):
    """Bit-exact, NaNs compared as a class (reading R7)."""
    got, want = np.asarray(got), np.asarray(want)
    assert got.shape == want.shape and got.dtype == want.dtype, what
    if got.dtype == np.float32:
        gn, wn = np.isnan(got), np.isnan(want)
    else:
        gn = ((got & 0x7F80) == 0x7F80) & ((got & 0x7F) != 0)
        wn = ((want & 0x7F80) == 0x7F80) & ((want & 0x7F) != 0)
    assert np.array_equal(gn, wn), f"{what}: NaN positions differ"
    ok = gn | (bits(got) == bits(want))
    if not ok.all():
        bad = np.flatnonzero(~ok)
        raise AssertionError(f"{what}: {bad.size} of {got.size} words differ; first at {bad[:5]}: "
                             f"got {got[bad[:5]]} want {want[bad[:5]]}")


def reduce_g1(xs_per_bucket, A=16, borrow_last=True, override=None, stash_dtypes=None, repeat=1, batched=False):
    """G = 1.  xs_per_bucket: list over buckets of lists over ESTs of arrays.
    stash_dtypes: optional per-bucket dtype of the *gradient* handed to the
    stash (a cast happens when it differs from the bucket dtype)."""
    N = len(xs_per_bucket[0])
    buckets = [(x[0].size, code(x[0])) for x in xs_per_bucket]
    agg = Aggregator(N, 1, 0, [0] * N, buckets, chunk_align=A)
    if override:
        agg.set_launch_override(*override)
    devs = []
    for b, xs in enumerate(xs_per_bucket):
        row = []
        for x in xs:
            if stash_dtypes and stash_dtypes[b] != code(x):
                t = to_dev(x)
                row.append(t.float() if stash_dtypes[b] == "f32" else t.to(torch.bfloat16))
            else:
                row.append(to_dev(x))
        devs.append(row)
    outs = [agg.new_out(b) for b in range(len(buckets))]
    results = []
    for _ in range(repeat):
        for k in range(N):
            if batched:
                mode = es.ES_STASH_BORROW if borrow_last and k == N - 1 else es.ES_STASH_COPY
                agg.stash_many(k, range(len(buckets)), [devs[b][k] for b in range(len(buckets))], mode)
                continue
            for b in range(len(buckets)):
                mode = es.ES_STASH_BORROW if (borrow_last and k == N - 1 and devs[b][k].dtype == outs[b].dtype) \
                    else es.ES_STASH_COPY
                agg.stash(k, b, devs[b][k], mode)
        if batched:
            agg.allreduce_many(range(len(buckets)), outs)
        else:
            for b in range(len(buckets)):
                agg.allreduce(b, outs[b])
        torch.cuda.synchronize()
        agg.sync()
        results.append([from_dev(o) for o in outs])
    agg.close()
    return results if repeat > 1 else results[0]


def reduce_loopback(xs_per_bucket, G, mapping, sched=es.ES_SCHED_AUTO, A=16, borrow_last=True, steps=1,
                    batched=False, options=0):
    """G ranks in one process over the LOOPBACK transport, one host thread and
    one CUDA stream per rank, all on the current GPU.  Returns per-rank lists
    of outputs (each rank must hold the full averaged buckets)."""
    N = len(xs_per_bucket[0])
    buckets = [(x[0].size, code(x[0])) for x in xs_per_bucket]
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, g, mapping, buckets, chunk_align=A, transport=es.ES_TRANSPORT_LOOPBACK,
                       comm=world.value, sched=sched, options=options) for g in range(G)]
    if sched in es.PEER_SCHEDS:                   # same process: peers map by raw address
        blobs = [a.peer_blob() for a in aggs]
        for a in aggs:
            a.peer_open(blobs)
    devs = [[to_dev(x) for x in xs] for xs in xs_per_bucket]
    outs = [[a.new_out(b) for b in range(len(buckets))] for a in aggs]
    streams = [torch.cuda.Stream() for _ in range(G)]
    torch.cuda.synchronize()
    errors = []
    dev_index = torch.cuda.current_device()

    def run(g):
        try:
            torch.cuda.set_device(dev_index)
            a = aggs[g]
            with torch.cuda.stream(streams[g]):
                for _ in range(steps):
                    loc = a.local_ests
                    for i, k in enumerate(loc):
                        mode = es.ES_STASH_BORROW if (borrow_last and i == len(loc) - 1) else es.ES_STASH_COPY
                        if options & es.ES_OPT_INCREMENTAL:      # NEXT-1: fold at the stash
                            a.stash_fold(k, range(len(buckets)), [devs[b][k] for b in range(len(buckets))], mode)
                        elif batched:
                            a.stash_many(k, range(len(buckets)), [devs[b][k] for b in range(len(buckets))], mode)
                        else:
                            for b in range(len(buckets)):
                                a.stash(k, b, devs[b][k], mode)
                    if batched:
                        a.allreduce_many(range(len(buckets)), outs[g])
                    else:
                        for b in range(len(buckets)):
                            a.allreduce(b, outs[g][b])
        except Exception as e:  # surfaced below
            errors.append((g, e))

    ths = [threading.Thread(target=run, args=(g,)) for g in range(G)]
    for t in ths:
        t.start()
    for t in ths:
        t.join(timeout=300)
    torch.cuda.synchronize()
    if errors:
        raise errors[0][1]
    res = [[from_dev(o) for o in outs[g]] for g in range(G)]
    for a in aggs:
        a.sync()
        a.close()
    es.es_loopback_destroy(world)
    return res


def check_whole_output(what, outs, fetch, buckets, N, win=1 << 21):
    """The WHOLE reduced bucket set against the oracle (plain definition, windows of `win`
    elements on a thread pool: the C oracle releases the GIL), bit-exact.  fetch(k, b) -> EST
    k's bucket b as a host array."""
    import concurrent.futures as cf
    import os

    import oracle
    host = [[fetch(k, b) for k in range(N)] for b in range(len(buckets))]
    got = [from_dev(o) for o in outs]
    jobs = [(b, s, min(win, L - s)) for b, (L, _) in enumerate(buckets) for s in range(0, L, win)]

    def run(j):
        b, s, n = j
        L, d = buckets[b]
        want = oracle.reduce([host[b][k][s:s + n] for k in range(N)], d, L=L, first=s)
        assert_bits_equal(got[b][s:s + n], want, f"{what} b={b} s={s}")
        return n
    with cf.ThreadPoolExecutor(max_workers=len(os.sched_getaffinity(0))) as ex:
        assert sum(ex.map(run, jobs)) == sum(L for L, _ in buckets)
