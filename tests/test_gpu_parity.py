"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
bit for bit (readings R1-R7; north star: "The GPU result must match the
oracle bit-exactly").  Sizes span several tiles and ragged tails; the
full-size sampled checks run in the launch configuration bench.py times."""
import json
import os

import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads

from gpu_util import assert_bits_equal, reduce_g1, reduce_loopback

pytestmark = pytest.mark.gpu


def _bf16(x32):
    return oracle.f32_to_bf16_bits(np.asarray(x32, np.float32))


def _gauss(rng, N, L, dtype="f32", sigma=1e-3):
    mu = rng.standard_normal(L) * sigma
    xs = [(mu + rng.standard_normal(L) * sigma).astype(np.float32) for _ in range(N)]
    return xs if dtype == "f32" else [_bf16(x) for x in xs]


# ---- G = 1 -----------------------------------------------------------------------------------

@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("N", [1, 2, 3, 4, 8, 12, 16, 32, 33, 129])
def test_fold_g1_matches_oracle(N, dtype):
    rng = np.random.default_rng(N * 7 + (dtype == "bf16"))
    Ls = [100003, 16, 17, 1, 4099]                   # several tiles + ragged tails
    xs = [_gauss(rng, N, L, dtype) for L in Ls]
    outs = reduce_g1(xs)
    for b, L in enumerate(Ls):
        assert_bits_equal(outs[b], oracle.reduce(xs[b], dtype), f"N={N} L={L} {dtype}")


@pytest.mark.parametrize("N", [3, 8, 32])
def test_batched_api_mixed_dtypes(N):
    """es_stash_grads / es_allreduce_many: many buckets (mixed fp32 / bf16,
    ragged, empty) per multi-segment launch give the oracle's bits."""
    rng = np.random.default_rng(300 + N)
    Ls = [100003, 16, 0, 17, 65536, 4099, 1, 2049000 // 8]
    dts = ["f32", "bf16", "f32", "bf16", "bf16", "f32", "f32", "f32"]
    xs = [_gauss(rng, N, L, d) for L, d in zip(Ls, dts)]
    for batched in (True, False):
        outs = reduce_g1(xs, batched=batched)
        for b, (L, d) in enumerate(zip(Ls, dts)):
            assert_bits_equal(outs[b], oracle.reduce(xs[b], d), f"batched={batched} N={N} b={b}")


def test_batched_launch_shapes():
    rng = np.random.default_rng(301)
    xs = [_gauss(rng, 12, L) for L in (50001, 7, 300000, 129)]
    want = [oracle.reduce(x, "f32") for x in xs]
    for ov in [(4, 32), (5, 256), (64, 64), (2000, 128), (0, 0)]:
        outs = reduce_g1(xs, batched=True, override=ov)
        for b in range(4):
            assert_bits_equal(outs[b], want[b], f"override {ov} b={b}")


@pytest.mark.parametrize("L", [0, 1, 15, 16, 17, 1000003])
def test_fold_g1_tails(L):
    rng = np.random.default_rng(L)
    for dtype in ["f32", "bf16"]:
        xs = _gauss(rng, 4, max(L, 1), dtype)
        if L == 0:
            xs = [x[:0] for x in xs]
        out = reduce_g1([xs])[0]
        assert_bits_equal(out, oracle.reduce(xs, dtype), f"L={L} {dtype}")


@pytest.mark.parametrize("A", [8, 16, 64, 4096])
def test_fold_g1_chunk_align(A):
    rng = np.random.default_rng(A)
    xs = _gauss(rng, 7, 50001)
    assert_bits_equal(reduce_g1([xs], A=A)[0], oracle.reduce(xs, "f32", A=A), f"A={A}")


def test_golden_witnesses_on_gpu(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "witness_n4.json")))
    for case in g["cases"]:
        xs = [np.full(g["L"], np.float32(float.fromhex(v) if "0x" in v else float(v)), np.float32) for v in case["x"]]
        assert_bits_equal(reduce_g1([xs], A=g["A"])[0], oracle.reduce(xs, "f32", A=g["A"]), case["name"])
    b = json.load(open(os.path.join(golden_dir, "bf16_accumulate.json")))
    xs = [_bf16(np.full(b["L"], np.float32(float.fromhex(v) if "0x" in v else float(v)))) for v in b["x"]]
    out = reduce_g1([xs], A=b["A"])[0]
    assert np.all(oracle.bf16_bits_to_f32(out) == np.float32(float(b["out"])))


def test_special_values_on_gpu():
    t = np.float32(2.0 ** -149)
    cases = [
        [np.full(64, -0.0, np.float32)] * 4,                                    # R3 signed zero
        [np.full(64, 2 * t, np.float32), np.full(64, 4 * t, np.float32)],      # subnormals (no FTZ)
        [np.full(64, 1.0, np.float32), np.full(64, np.nan, np.float32), np.full(64, 2.0, np.float32)],
        [np.full(64, np.inf, np.float32), np.full(64, -np.inf, np.float32)],
        [np.array([0.0, -0.0, 1.5, np.inf, -np.inf, 1e-45, 3.4e38, np.nan] * 8, np.float32)],  # N = 1 identity
    ]
    for xs in cases:
        assert_bits_equal(reduce_g1([xs])[0], oracle.reduce(xs, "f32"))
        xb = [_bf16(x) for x in xs]
        assert_bits_equal(reduce_g1([xb])[0], oracle.reduce(xb, "bf16"))


def test_wide_dynamic_range():
    rng = np.random.default_rng(99)
    N, L = 12, 70001
    xs = [(rng.choice([-1, 1], L) * 2.0 ** rng.uniform(-20, 20, L)).astype(np.float32) for _ in range(N)]
    assert_bits_equal(reduce_g1([xs])[0], oracle.reduce(xs, "f32"))


def test_launch_config_invariance():
    """T4 / D2 analogue: grid and block size never change bits."""
    rng = np.random.default_rng(4)
    xs_f = _gauss(rng, 12, 123457)
    xs_b = _gauss(rng, 12, 123457, "bf16")
    ref_f, ref_b = oracle.reduce(xs_f, "f32"), oracle.reduce(xs_b, "bf16")
    for ov in [(1, 32), (1, 256), (3, 64), (148, 128), (1184, 256), (7, 96), (0, 0)]:
        out = reduce_g1([xs_f, xs_b], override=ov)
        assert_bits_equal(out[0], ref_f, f"override {ov}")
        assert_bits_equal(out[1], ref_b, f"override {ov}")


def test_repeatability_d0():
    """D0: repeated runs give identical bits."""
    rng = np.random.default_rng(5)
    xs = _gauss(rng, 8, 300001)
    runs = reduce_g1([xs], repeat=10)
    for r in runs[1:]:
        assert_bits_equal(r[0], runs[0][0])
    assert_bits_equal(runs[0][0], oracle.reduce(xs, "f32"))


def test_layout_dependence_negative():
    """D0 failure mode: a different bucket layout (here a
    different chunk alignment, part of the persisted layout) changes bits --
    the suite detects layout dependence."""
    rng = np.random.default_rng(6)
    xs = _gauss(rng, 8, 200003)
    a = reduce_g1([xs], A=16)[0]
    b = reduce_g1([xs], A=1024)[0]
    assert not np.array_equal(a.view(np.uint32), b.view(np.uint32))


# ---- stash -------------------------------------------------------------------------------

@pytest.mark.parametrize("src,dst", [("f32", "f32"), ("f32", "bf16"), ("bf16", "f32"), ("bf16", "bf16")])
def test_stash_cast_parity(src, dst):
    """Stash = cast (RNE narrowing, exact widening) then fold: the fold of
    the cast slots must equal the oracle's fold of the oracle's cast."""
    rng = np.random.default_rng(8)
    N, L = 5, 65541
    base = _gauss(rng, N, L, src, sigma=10.0)
    oracle_slots = [oracle.stash(x, src, dst) for x in base]
    # hand the kernel `src`-typed gradients for a `dst` bucket
    from gpu_util import Aggregator, to_dev, from_dev
    agg = Aggregator(N, 1, 0, [0] * N, [(L, dst)])
    devs = [to_dev(x) for x in base]
    for k in range(N):
        agg.stash(k, 0, devs[k], es.ES_STASH_COPY)
    o = agg.new_out(0)
    agg.allreduce(0, o)
    torch.cuda.synchronize()
    agg.sync()
    assert_bits_equal(from_dev(o), oracle.reduce(oracle_slots, dst), f"{src}->{dst}")
    agg.close()


def test_borrow_equals_copy_and_out_aliasing():
    rng = np.random.default_rng(9)
    xs = _gauss(rng, 6, 77777)
    want = oracle.reduce(xs, "f32")
    assert_bits_equal(reduce_g1([xs], borrow_last=False)[0], want)
    assert_bits_equal(reduce_g1([xs], borrow_last=True)[0], want)
    # out aliases the borrowed buffer of the last EST (in-place)
    from gpu_util import Aggregator, to_dev, from_dev
    agg = Aggregator(6, 1, 0, [0] * 6, [(77777, "f32")])
    devs = [to_dev(x) for x in xs]
    for k in range(5):
        agg.stash(k, 0, devs[k])
    agg.stash(5, 0, devs[5], es.ES_STASH_BORROW)
    agg.allreduce(0, devs[5])
    torch.cuda.synchronize()
    assert_bits_equal(from_dev(devs[5]), want)
    agg.close()


@pytest.mark.parametrize("options", [0, es.ES_OPT_STASH_BACKGROUND])
def test_per_bucket_allreduce_interleaved_with_last_stashes(options):
    """DDP-style bucket overlap (profiles/r01_overlap.md, +bk): the last EST stashes bucket b and
    es_allreduce(b) runs at once, before its later buckets exist; earlier ESTs stash per bucket
    on a side stream in the order their buckets become ready.  Every bucket equals the oracle."""
    from gpu_util import Aggregator, to_dev, from_dev
    rng = np.random.default_rng(21)
    N = 5
    sizes = [(40003, "f32"), (777, "bf16"), (123457, "f32"), (16, "bf16")]
    xs = [_gauss(rng, N, L, d) for L, d in sizes]
    agg = Aggregator(N, 1, 0, [0] * N, sizes, options=options)
    side = torch.cuda.Stream()
    outs = [agg.new_out(b) for b in range(len(sizes))]
    devs = [[to_dev(xs[b][k]) for b in range(len(sizes))] for k in range(N)]
    torch.cuda.synchronize()
    with torch.cuda.stream(side):
        for k in range(N):
            for b in range(len(sizes)):
                if k < N - 1:
                    agg.stash(k, b, devs[k][b])
                else:
                    agg.stash(k, b, devs[k][b], es.ES_STASH_BORROW)
                    agg.allreduce(b, outs[b])
    torch.cuda.synchronize()
    agg.sync()
    for b, (L, d) in enumerate(sizes):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], d), f"bucket {b}")
    agg.close()


# ---- G > 1 over the loopback transport (one GPU, every mapping) ------------------------------

def _surjections(N, G):
    import itertools
    for m in itertools.product(range(G), repeat=N):
        if len(set(m)) == G:
            yield list(m)


@pytest.mark.parametrize("G", [2, 3, 4])
def test_all_mappings_n4_loopback(G):
    rng = np.random.default_rng(40 + G)
    xs = [_gauss(rng, 4, 1001), _gauss(rng, 4, 64, "bf16"), _gauss(rng, 4, 3)]
    want = [oracle.reduce(xs[0], "f32"), oracle.reduce(xs[1], "bf16"), oracle.reduce(xs[2], "f32")]
    for m in _surjections(4, G):
        for sched in (es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN, es.ES_SCHED_PEER, es.ES_SCHED_PEER_CHAIN):
            res = reduce_loopback(xs, G, m, sched)
            for g in range(G):
                for b in range(3):
                    assert_bits_equal(res[g][b], want[b], f"map={m} sched={sched} rank={g} bucket={b}")


@pytest.mark.parametrize("G,kind", [(2, "contiguous"), (4, "contiguous"), (8, "contiguous"), (8, "round_robin"),
                                    (4, "random"), (8, "random"), (3, "random")])
@pytest.mark.parametrize("sched", [es.ES_SCHED_AUTO, es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN, es.ES_SCHED_PEER,
                                   es.ES_SCHED_PEER_CHAIN, es.ES_SCHED_PEER_AUTO])
def test_mappings_n8_loopback(G, kind, sched):
    rng = np.random.default_rng(G * 10 + len(kind))
    xs = [_gauss(rng, 8, 200003), _gauss(rng, 8, 4096 + 5, "bf16")]
    want = [oracle.reduce(xs[0], "f32"), oracle.reduce(xs[1], "bf16")]
    res = reduce_loopback(xs, G, workloads.mapping(8, G, kind), sched)
    for g in range(G):
        for b in range(2):
            assert_bits_equal(res[g][b], want[b], f"G={G} {kind} sched={sched} rank={g} b={b}")


@pytest.mark.parametrize("G,kind", [(2, "contiguous"), (4, "random"), (8, "contiguous"), (8, "round_robin"),
                                    (3, "random")])
@pytest.mark.parametrize("sched,options", [(es.ES_SCHED_PEER, 0), (es.ES_SCHED_PEER_AUTO, 0),
                                           (es.ES_SCHED_PEER_CHAIN, es.ES_OPT_PEER_ROUNDS),
                                           (es.ES_SCHED_PEER_CHAIN, 0)])
@pytest.mark.parametrize("batched", [False, True])
def test_peer_push_loopback(G, kind, sched, options, batched):
    """ES_OPT_PEER_PUSH: owners push their finished shards / chunks into every peer's RESULT area
    inside the fold; gathers read the own RESULT.  Repeated steps (RESULT reuse across steps and
    buckets) keep the oracle's bits on every rank.  PEER_CHAIN without PEER_ROUNDS (k_fold_pipe)
    ignores the option and must be unaffected."""
    rng = np.random.default_rng(700 + G * 10 + len(kind))
    xs = [_gauss(rng, 8, 200003), _gauss(rng, 8, 4096 + 5, "bf16"), _gauss(rng, 8, 17)]
    want = [oracle.reduce(xs[0], "f32"), oracle.reduce(xs[1], "bf16"), oracle.reduce(xs[2], "f32")]
    res = reduce_loopback(xs, G, workloads.mapping(8, G, kind), sched, steps=3, batched=batched,
                          options=options | es.ES_OPT_PEER_PUSH)
    for g in range(G):
        for b in range(3):
            assert_bits_equal(res[g][b], want[b], f"push G={G} {kind} sched={sched} opt={options} rank={g} b={b}")


@pytest.mark.parametrize("kind", ["contiguous", "round_robin"])
def test_bert_uneven_n12_g8_loopback(kind):
    """BERT config shape: N=12 on G=8, n = [2,2,2,2,1,1,1,1] (contiguous) and
    k mod 8 (round robin): identical bits, equal to the oracle and to G=1."""
    rng = np.random.default_rng(12)
    xs = [_gauss(rng, 12, 120011, "bf16"), _gauss(rng, 12, 30000, "bf16")]
    want = [oracle.reduce(x, "bf16") for x in xs]
    g1 = reduce_g1(xs)
    res = reduce_loopback(xs, 8, workloads.mapping(12, 8, kind))
    for b in range(2):
        assert_bits_equal(g1[b], want[b])
        for g in range(8):
            assert_bits_equal(res[g][b], want[b], f"{kind} rank={g} b={b}")


@pytest.mark.parametrize("sched", [es.ES_SCHED_CHAIN, es.ES_SCHED_DIRECT, es.ES_SCHED_PEER, es.ES_SCHED_PEER_CHAIN])
@pytest.mark.parametrize("batched", [False, True])
def test_loopback_multi_step_reuse(sched, batched):
    """Three global steps on the same handles: slot / staging / partial reuse is ordered."""
    rng = np.random.default_rng(13)
    xs = [_gauss(rng, 8, 50001), _gauss(rng, 8, 70001), _gauss(rng, 8, 3001, "bf16")]
    want = [oracle.reduce(x, d) for x, d in zip(xs, ["f32", "f32", "bf16"])]
    res = reduce_loopback(xs, 4, workloads.mapping(8, 4, "random"), sched, steps=3, batched=batched)
    for g in range(4):
        for b in range(3):
            assert_bits_equal(res[g][b], want[b])


# ---- full size, in the bench launch configuration: sampled windows -----------------------------

def _bench_step(agg, local, grads, outs, incremental=False):
    """Exactly bench.py's step: switch-in, fused stash+switch per EST, the last
    local EST borrowed, one batched allreduce (incremental: bench.py's NEXT-1
    leg -- switch, es_stash_fold_grads per EST)."""
    B = len(outs)
    if incremental:
        for i, k in enumerate(local):
            agg.switch(k)
            agg.stash_fold(k, range(B), grads[k], es.ES_STASH_BORROW if i == len(local) - 1 else es.ES_STASH_COPY)
        agg.allreduce_many(range(B), outs)
        return
    agg.switch(local[0])
    for i, k in enumerate(local):
        if i == len(local) - 1:
            agg.stash_many(k, range(B), grads[k], es.ES_STASH_BORROW)
        else:
            agg.stash_and_switch(k, range(B), grads[k], local[i + 1], es.ES_STASH_COPY)
    agg.allreduce_many(range(B), outs)


def _check_sampled(name, outs, fetch, buckets, N, seed=0):
    from gpu_util import from_dev
    rng = np.random.default_rng(seed)
    for b, (L, d) in enumerate(buckets):
        C = oracle.chunk_elems(L, N)
        starts = [0, max(0, L - 4099), max(0, C - 2000), max(0, (N - 1) * C - 7)] + \
            list(rng.integers(0, max(1, L - 4099), 3))
        for s in starts:
            s = int(min(s, L - 1))
            n = min(4099, L - s)
            want = oracle.reduce([fetch(k, b, s, n) for k in range(N)], d, L=L, first=s)
            assert_bits_equal(from_dev(outs[b][s:s + n]), want, f"{name} b={b} s={s}")


@pytest.mark.parametrize("name", ["tiny", "resnet50", "vgg19", "bert_base", "swin_b"])
def test_full_size_whole_output_parity(name):
    """BASELINE.json's full sizes at G=1, in bench.py's launch configuration
    (CUDA graph of the fused step, replayed): the WHOLE output against the
    oracle (all host cores), plus sampled windows at chunk boundaries and the
    ragged end, plus a property at any size."""
    from gpu_util import check_whole_output
    cfg = workloads.config(name)
    N = cfg["N"]
    from gpu_util import Aggregator, from_dev
    buckets = cfg["buckets"]
    agg = Aggregator(N, 1, 0, [0] * N, buckets, state_nbytes=workloads.state_nbytes())
    live = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in workloads.state_nbytes()]
    agg.register_state(live)
    for k in range(N):
        for i, blob in enumerate(workloads.est_state(name, k)):
            agg.init_state(k, i, blob)
    grads = {k: [workloads.est_bucket(name, k, b, device="cuda") for b in range(len(buckets))] for k in range(N)}
    outs = [agg.new_out(b) for b in range(len(buckets))]
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        _bench_step(agg, list(range(N)), grads, outs)        # eager warm-up
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        _bench_step(agg, list(range(N)), grads, outs)
    for o in outs:
        o.zero_()
    for _ in range(2):
        g.replay()
    torch.cuda.synchronize()
    agg.sync()
    _check_sampled(name, outs, lambda k, b, st, n: from_dev(grads[k][b][st:st + n]), buckets, N)
    check_whole_output(name, outs, lambda k, b: from_dev(grads[k][b]), buckets, N)
    for b in range(len(buckets)):         # property at any size: finite, |out| <= max_k |x_k| (+ rounding)
        o = outs[b].float()
        mx = grads[0][b].float().abs()
        for k in range(1, N):
            mx = torch.maximum(mx, grads[k][b].float().abs())
        assert torch.isfinite(o).all() and bool((o.abs() <= mx * 1.01).all())
    agg.close()


@pytest.mark.parametrize("name,G,kind,inc", [("resnet50", 8, "contiguous", False), ("resnet50", 2, "contiguous", False),
                                             ("bert_base", 8, "contiguous", False),
                                             ("bert_base", 8, "round_robin", False),
                                             ("vgg19", 4, "contiguous", False), ("swin_b", 4, "contiguous", True),
                                             ("bert_base", 8, "contiguous", True)])
def test_full_size_multi_rank_loopback(name, G, kind, inc):
    """The configs' G > 1 shapes at full size over the loopback transport
    (all G ranks on this GPU; AUTO: tile-pipelined CHAIN / DIRECT): every rank
    holds the oracle's bits (rank 0's whole output checked).  inc: NEXT-1."""
    import threading
    cfg = workloads.config(name)
    N = cfg["N"]
    from gpu_util import Aggregator, from_dev
    buckets = cfg["buckets"]
    m = workloads.mapping(N, G, kind)
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, r, m, buckets, state_nbytes=workloads.state_nbytes(),
                       transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value,
                       options=es.ES_OPT_INCREMENTAL if inc else 0) for r in range(G)]
    lives = []
    for r, a in enumerate(aggs):
        live = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in workloads.state_nbytes()]
        a.register_state(live)
        lives.append(live)
        for k in a.local_ests:
            for i, blob in enumerate(workloads.est_state(name, k)):
                a.init_state(k, i, blob)
    grads = {k: [workloads.est_bucket(name, k, b, device="cuda") for b in range(len(buckets))] for k in range(N)}
    outs = [[a.new_out(b) for b in range(len(buckets))] for a in aggs]
    streams = [torch.cuda.Stream() for _ in range(G)]
    torch.cuda.synchronize()
    errs = []

    def run(r):
        try:
            with torch.cuda.stream(streams[r]):
                _bench_step(aggs[r], aggs[r].local_ests, grads, outs[r], incremental=inc)
        except Exception as e:
            errs.append(e)
    ts = [threading.Thread(target=run, args=(r,)) for r in range(G)]
    [t.start() for t in ts]
    [t.join(timeout=600) for t in ts]
    torch.cuda.synchronize()
    if errs:
        raise errs[0]
    fetch = lambda k, b, st, n: from_dev(grads[k][b][st:st + n])  # noqa: E731
    for r in (0, G - 1):
        _check_sampled(f"{name} G={G} {kind} rank {r}", outs[r], fetch, buckets, N, seed=r)
    from gpu_util import check_whole_output
    check_whole_output(f"{name} G={G} {kind} rank 0", outs[0], lambda k, b: from_dev(grads[k][b]), buckets, N)
    for r in range(1, G):                 # every rank holds the same bits
        for b in range(len(buckets)):
            iv = torch.int16 if outs[r][b].dtype == torch.bfloat16 else torch.int32
            assert torch.equal(outs[r][b].view(iv), outs[0][b].view(iv)), (r, b)
    for a in aggs:
        a.close()
    es.es_loopback_destroy(world)


# ---- NEXT-3 compatibility variants -------------------------------------------------------------

COMPATS = [es.ES_COMPAT_PREDIV, es.ES_COMPAT_PREMUL, es.ES_COMPAT_BF16_HOP,
           es.ES_COMPAT_PREDIV | es.ES_COMPAT_BF16_HOP, es.ES_COMPAT_PREMUL | es.ES_COMPAT_BF16_HOP]


@pytest.mark.parametrize("compat", COMPATS)
@pytest.mark.parametrize("N", [3, 12, 16])
def test_compat_variants_g1(compat, N):
    from gpu_util import Aggregator, from_dev, to_dev
    rng = np.random.default_rng(600 + N + compat)
    Ls, dts = [50003, 17, 4096], ["f32", "bf16", "bf16"]
    xs = [_gauss(rng, N, L, d, sigma=1.0) for L, d in zip(Ls, dts)]
    agg = Aggregator(N, 1, 0, [0] * N, list(zip(Ls, dts)), compat=compat)
    devs = [[to_dev(xs[b][k]) for b in range(3)] for k in range(N)]
    for k in range(N):
        agg.stash_many(k, range(3), devs[k], es.ES_STASH_BORROW if k == N - 1 else es.ES_STASH_COPY)
    outs = [agg.new_out(b) for b in range(3)]
    agg.allreduce_many(range(3), outs)
    torch.cuda.synchronize()
    for b in range(3):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce_ex(xs[b], dts[b], compat), f"compat={compat} b={b}")
    agg.close()


@pytest.mark.parametrize("sched", [es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN])
def test_compat_variants_loopback(sched):
    """Chain partials carry the variant's (bf16-rounded) value between GPUs."""
    rng = np.random.default_rng(700)
    for compat in COMPATS:
        xs = [_gauss(rng, 12, 30001, "bf16", sigma=1.0), _gauss(rng, 12, 999, "f32", sigma=1.0)]
        want = [oracle.reduce_ex(xs[0], "bf16", compat), oracle.reduce_ex(xs[1], "f32", compat)]
        from gpu_util import Aggregator, from_dev, to_dev  # noqa: F401
        res = _loopback_compat(xs, 4, workloads.mapping(12, 4, "random", seed=compat), sched, compat)
        for g in range(4):
            for b in range(2):
                assert_bits_equal(res[g][b], want[b], f"compat={compat} sched={sched} rank={g} b={b}")


def _loopback_compat(xs_per_bucket, G, mapping, sched, compat):
    import threading
    from gpu_util import Aggregator, code, from_dev, to_dev
    N = len(xs_per_bucket[0])
    buckets = [(x[0].size, code(x[0])) for x in xs_per_bucket]
    world = es.es_loopback_create(G)
    aggs = [Aggregator(N, G, g, mapping, buckets, transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value,
                       sched=sched, compat=compat) for g in range(G)]
    devs = [[to_dev(x) for x in xs] for xs in xs_per_bucket]
    outs = [[a.new_out(b) for b in range(len(buckets))] for a in aggs]
    streams = [torch.cuda.Stream() for _ in range(G)]
    torch.cuda.synchronize()
    errs = []

    def run(g):
        try:
            with torch.cuda.stream(streams[g]):
                for k in aggs[g].local_ests:
                    aggs[g].stash_many(k, range(len(buckets)), [devs[b][k] for b in range(len(buckets))])
                aggs[g].allreduce_many(range(len(buckets)), outs[g])
        except Exception as e:
            errs.append(e)
    ts = [threading.Thread(target=run, args=(g,)) for g in range(G)]
    [t.start() for t in ts]
    [t.join(timeout=300) for t in ts]
    torch.cuda.synchronize()
    if errs:
        raise errs[0]
    res = [[from_dev(o) for o in row] for row in outs]
    for a in aggs:
        a.close()
    es.es_loopback_destroy(world)
    return res


# ---- NEXT-1 incremental canonical fold ---------------------------------------------------------

@pytest.mark.parametrize("N", [1, 2, 3, 8, 12, 32])
def test_incremental_fold_matches_oracle(N):
    from gpu_util import Aggregator, from_dev, to_dev
    rng = np.random.default_rng(900 + N)
    Ls, dts = [100003, 40, 4099, 1], ["f32", "bf16", "f32", "bf16"]     # 40 < N*C for N >= 3: empty chunks
    agg = Aggregator(N, 1, 0, [0] * N, list(zip(Ls, dts)), options=es.ES_OPT_INCREMENTAL)
    outs = [agg.new_out(b) for b in range(len(Ls))]
    for step in range(2):
        xs = [_gauss(rng, N, L, d) for L, d in zip(Ls, dts)]
        devs = [[to_dev(xs[b][k]) for b in range(len(Ls))] for k in range(N)]
        for k in range(N):
            agg.stash_fold(k, range(len(Ls)), devs[k], es.ES_STASH_BORROW if k == N - 1 else es.ES_STASH_COPY)
        agg.allreduce_many(range(len(Ls)), outs)
        torch.cuda.synchronize()
        for b, d in enumerate(dts):
            assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], d), f"step {step} N={N} b={b}")
    agg.close()


def test_incremental_fold_protocol_and_graph():
    from gpu_util import Aggregator, from_dev, to_dev
    N, L = 4, 5000
    rng = np.random.default_rng(901)
    xs = _gauss(rng, N, L)
    devs = [to_dev(x) for x in xs]
    agg = Aggregator(N, 1, 0, [0] * N, [(L, "f32")], options=es.ES_OPT_INCREMENTAL)
    out = agg.new_out(0)
    with pytest.raises(es.EsError) as e:              # must start with EST 0
        agg.stash_fold(1, [0], [devs[1]])
    assert e.value.status == es.ES_ESTATE
    agg.stash_fold(0, [0], [devs[0]])
    with pytest.raises(es.EsError) as e:              # no mixing with the plain stash
        agg.stash(1, 0, devs[1])
    assert e.value.status == es.ES_ESTATE
    agg.stash_fold(1, [0], [devs[1]])
    agg.stash_fold(2, [0], [devs[2]])
    with pytest.raises(es.EsError) as e:              # incomplete: EST 3 has not run
        agg.allreduce(0, out)
    assert e.value.status == es.ES_ESTATE
    agg.stash_fold(3, [0], [devs[3]])
    agg.allreduce(0, out)
    torch.cuda.synchronize()
    assert_bits_equal(from_dev(out), oracle.reduce(xs, "f32"))
    # the whole incremental step as a CUDA graph
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for k in range(N):
            agg.stash_fold(k, [0], [devs[k]])
        agg.allreduce(0, out)
    out.zero_()
    g.replay()
    g.replay()
    torch.cuda.synchronize()
    assert_bits_equal(from_dev(out), oracle.reduce(xs, "f32"))
    agg.close()


def _inc_want(xs, dts):
    return [oracle.reduce(x, d) for x, d in zip(xs, dts)]


@pytest.mark.parametrize("G,kind", [(2, "contiguous"), (4, "contiguous"), (8, "contiguous"), (2, "round_robin"),
                                    (4, "round_robin"), (8, "round_robin"), (2, "random"), (4, "random"),
                                    (3, "random")])
@pytest.mark.parametrize("sched", [es.ES_SCHED_AUTO, es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN, es.ES_SCHED_PEER,
                                   es.ES_SCHED_PEER_CHAIN, es.ES_SCHED_PEER_AUTO])
def test_incremental_fold_loopback_n8(G, kind, sched):
    """NEXT-1 at G > 1: every rank folds the local prefix of each sequence that
    starts on it (chain first segments, the local run opening a DIRECT/PEER
    shard fold) into fp32 partials at the stashes; the end fold continues from
    them.  Two steps on the same handles (partials reused), oracle bits on
    every rank, for every schedule and mapping kind."""
    rng = np.random.default_rng(1500 + G * 10 + len(kind))
    dts = ["f32", "bf16", "f32"]
    xs = [_gauss(rng, 8, 200003), _gauss(rng, 8, 4096 + 5, "bf16"), _gauss(rng, 8, 40)]
    res = reduce_loopback(xs, G, workloads.mapping(8, G, kind), sched, steps=2,
                          options=es.ES_OPT_INCREMENTAL)
    want = _inc_want(xs, dts)
    for g in range(G):
        for b in range(3):
            assert_bits_equal(res[g][b], want[b], f"inc G={G} {kind} sched={sched} rank={g} b={b}")


@pytest.mark.parametrize("kind", ["contiguous", "round_robin"])
@pytest.mark.parametrize("sched", [es.ES_SCHED_AUTO, es.ES_SCHED_PEER_AUTO, es.ES_SCHED_CHAIN,
                                   es.ES_SCHED_PEER_CHAIN])
def test_incremental_fold_bert_n12_g8(kind, sched):
    """NEXT-1 on the BERT shape: N=12 bf16 on G=8, uneven n_g, both maps."""
    rng = np.random.default_rng(1600 + len(kind))
    xs = [_gauss(rng, 12, 120011, "bf16"), _gauss(rng, 12, 30000, "bf16")]
    res = reduce_loopback(xs, 8, workloads.mapping(12, 8, kind), sched, steps=2, options=es.ES_OPT_INCREMENTAL)
    want = _inc_want(xs, ["bf16", "bf16"])
    for g in range(8):
        for b in range(2):
            assert_bits_equal(res[g][b], want[b], f"inc bert {kind} sched={sched} rank={g} b={b}")


@pytest.mark.parametrize("G", [2, 3, 4])
def test_incremental_fold_all_maps_n4(G):
    """Every surjective map of N=4 onto G ranks, AUTO and PEER_AUTO, with NEXT-1."""
    rng = np.random.default_rng(1700 + G)
    xs = [_gauss(rng, 4, 1000), _gauss(rng, 4, 77, "bf16")]
    want = _inc_want(xs, ["f32", "bf16"])
    for m in _surjections(4, G):
        for sched in (es.ES_SCHED_AUTO, es.ES_SCHED_PEER_AUTO):
            res = reduce_loopback(xs, G, m, sched, options=es.ES_OPT_INCREMENTAL)
            for g in range(G):
                for b in range(2):
                    assert_bits_equal(res[g][b], want[b], f"inc map={m} sched={sched} rank={g} b={b}")


def test_incremental_fold_g2_protocol():
    """G > 1: local ESTs must come in ascending order; a remote EST is refused."""
    from gpu_util import Aggregator, to_dev
    L = 5000
    world = es.es_loopback_create(2)
    agg = Aggregator(4, 2, 0, [0, 0, 1, 1], [(L, "f32")], options=es.ES_OPT_INCREMENTAL,
                     transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value)
    x = to_dev(np.ones(L, np.float32))
    with pytest.raises(es.EsError) as e:              # EST 1 before EST 0
        agg.stash_fold(1, [0], [x])
    assert e.value.status == es.ES_ESTATE
    with pytest.raises(es.EsError) as e:              # EST 2 lives on rank 1
        agg.stash_fold(2, [0], [x])
    assert e.value.status == es.ES_ESTATE
    agg.close()
    es.es_loopback_destroy(world)


# ---- maximum sizes ----------------------------------------------------------------------------

def test_max_n_1024():
    """N at its limit (1024 ESTs -> 1024 source pointers in one launch)."""
    rng = np.random.default_rng(1024)
    xs = [_gauss(rng, 1024, 20011)]
    for batched in (False, True):
        assert_bits_equal(reduce_g1(xs, batched=batched)[0], oracle.reduce(xs[0], "f32"), f"batched={batched}")


@pytest.mark.parametrize("N", [1023, 1024])
def test_peer_push_at_the_pointer_table_limit(N):
    """ES_OPT_PEER_PUSH at G = 2: N = 1023 pushes (1023 sources + 1 push pointer fill the 1024-entry
    table), N = 1024 falls back to the pull gather on every rank (N + G - 1 > 1024)."""
    rng = np.random.default_rng(N)
    xs = [_gauss(rng, N, 4099)]
    m = workloads.mapping(N, 2, "round_robin")
    res = reduce_loopback(xs, 2, m, es.ES_SCHED_PEER, options=es.ES_OPT_PEER_PUSH)
    want = oracle.reduce(xs[0], "f32")
    for g in range(2):
        assert_bits_equal(res[g][0], want, f"N={N} rank={g}")


def test_max_bucket_numel_2p31_minus_1():
    """The largest legal bucket (2^31 - 1 elements, bf16, 4 GiB per EST): the
    32-bit chunk arithmetic and 64-bit offsets hold to the last element."""
    from gpu_util import Aggregator, from_dev
    L, N = (1 << 31) - 1, 3
    g = torch.Generator(device="cuda").manual_seed(31)
    xs = [(torch.randn(L, generator=g, device="cuda") * 1e-3).to(torch.bfloat16) for _ in range(N)]
    agg = Aggregator(N, 1, 0, [0] * N, [(L, "bf16")])
    for k in range(N):
        agg.stash(k, 0, xs[k], es.ES_STASH_BORROW if k == N - 1 else es.ES_STASH_COPY)
    out = agg.new_out(0)
    agg.allreduce(0, out)
    torch.cuda.synchronize()
    C = oracle.chunk_elems(L, N)
    for s in [0, C - 9, 2 * C - 5, L - 4099, (1 << 30) + 7]:
        n = min(4099, L - s)
        want = oracle.reduce([from_dev(x[s:s + n]) for x in xs], "bf16", L=L, first=s)
        assert_bits_equal(from_dev(out[s:s + n]), want, f"s={s}")
    agg.close()
    with pytest.raises(es.EsError):                     # 2^31 is refused
        es.es_workspace_bytes(es.Config(2, 1, 0, [0, 0], [(1 << 31, es.ES_BF16)]))


def test_sixteen_loopback_ranks():
    rng = np.random.default_rng(16)
    xs = [_gauss(rng, 40, 50021), _gauss(rng, 40, 999, "bf16")]
    want = [oracle.reduce(xs[0], "f32"), oracle.reduce(xs[1], "bf16")]
    res = reduce_loopback(xs, 16, workloads.mapping(40, 16, "random", seed=5), es.ES_SCHED_AUTO)
    for g in range(16):
        for b in range(2):
            assert_bits_equal(res[g][b], want[b], f"rank={g} b={b}")
    # peer schedules need a hardware queue per same-process rank: refused, never hung
    with pytest.raises(es.EsError) as e:
        reduce_loopback(xs, 16, workloads.mapping(40, 16, "random", seed=5), es.ES_SCHED_PEER_AUTO)
    assert e.value.status == es.ES_EUNSUPPORTED


# ---- PEER_CHAIN tile pipelining (k_fold_pipe) --------------------------------------------------

@pytest.mark.parametrize("options", [0, es.ES_OPT_PEER_ROUNDS])
@pytest.mark.parametrize("G,N,kind", [(2, 8, "contiguous"), (4, 8, "contiguous"), (3, 12, "random"),
                                      (8, 12, "contiguous"), (4, 16, "round_robin")])
def test_peer_chain_pipelined_many_tiles(options, G, N, kind):
    """Chunks of tens of k_fold_pipe tiles (8192 elements) plus ragged tails,
    mixed dtypes, three steps on the same handles: the tile-pipelined chain
    (per-tile flags instead of round barriers) and the round-barrier chain
    both give the oracle's bits on every rank."""
    rng = np.random.default_rng(1000 + G * N)
    xs = [_gauss(rng, N, 1_000_003), _gauss(rng, N, 262_147, "bf16"), _gauss(rng, N, 8195)]
    want = [oracle.reduce(xs[0], "f32"), oracle.reduce(xs[1], "bf16"), oracle.reduce(xs[2], "f32")]
    m = workloads.mapping(N, G, kind, seed=11)
    res = reduce_loopback(xs, G, m, es.ES_SCHED_PEER_CHAIN, steps=3, batched=True, options=options)
    for g in range(G):
        for b in range(3):
            assert_bits_equal(res[g][b], want[b], f"G={G} N={N} {kind} opt={options} rank={g} b={b}")


@pytest.mark.parametrize("options", [0, es.ES_OPT_PEER_ROUNDS, es.ES_OPT_INCREMENTAL])
@pytest.mark.parametrize("G,N,kind", [(2, 4, "contiguous"), (4, 4, "contiguous"), (3, 6, "random"),
                                      (2, 8, "round_robin")])
def test_chain_tile_pipelined_transport(options, G, N, kind):
    """CHAIN over a transport (loopback here, NCCL on a multi-GPU box): chunks of
    ~3 M elements are cut into W = 3 tiles whose folds (caller's stream) and
    partial transfers (the handle's side stream) run in wavefront order; the
    round executor (ES_OPT_PEER_ROUNDS) and NEXT-1 on top of the pipelined one
    give the same bits.  Two steps reuse the events, side stream and partials."""
    rng = np.random.default_rng(1400 + G * N + len(kind))
    L = N * (3 << 20) + 13
    xs = [_gauss(rng, N, L), _gauss(rng, N, N * (1 << 20) + 8, "bf16"), _gauss(rng, N, 100)]
    want = [oracle.reduce(xs[0], "f32"), oracle.reduce(xs[1], "bf16"), oracle.reduce(xs[2], "f32")]
    m = workloads.mapping(N, G, kind, seed=5)
    res = reduce_loopback(xs, G, m, es.ES_SCHED_CHAIN, steps=2, batched=True, options=options)
    for g in range(G):
        for b in range(3):
            assert_bits_equal(res[g][b], want[b], f"G={G} N={N} {kind} opt={options} rank={g} b={b}")


def test_peer_auto_mixed_pipelined():
    """PEER_AUTO mixes PEER and PEER_CHAIN buckets in one batched call; both
    share the pipelined step's two barriers."""
    rng = np.random.default_rng(77)
    N, G = 8, 4
    xs = [_gauss(rng, N, 400_001), _gauss(rng, N, 70_001, "bf16"), _gauss(rng, N, 5)]
    want = [oracle.reduce(xs[0], "f32"), oracle.reduce(xs[1], "bf16"), oracle.reduce(xs[2], "f32")]
    for kind in ("contiguous", "round_robin"):
        res = reduce_loopback(xs, G, workloads.mapping(N, G, kind), es.ES_SCHED_PEER_AUTO, steps=2, batched=True)
        for g in range(G):
            for b in range(3):
                assert_bits_equal(res[g][b], want[b], f"{kind} rank={g} b={b}")


# ---- randomized schedules ------------------------------------------------------------------------

SCHED_NAMES = {es.ES_SCHED_DIRECT: "direct", es.ES_SCHED_CHAIN: "chain", es.ES_SCHED_AUTO: "auto",
               es.ES_SCHED_PEER: "peer", es.ES_SCHED_PEER_CHAIN: "peer_chain",
               es.ES_SCHED_PEER_AUTO: "peer_auto"}


@pytest.mark.parametrize("seed", range(int(os.environ.get("ES_FUZZ_SEEDS", "40"))))
def test_random_schedules_mappings_layouts(seed):
    """Seeded random N, G, EST->GPU map (any surjection), bucket layout (empty,
    tiny, ragged, multi-tile; f32/bf16), chunk alignment, schedule and
    PEER_CHAIN executor, one to three steps: every rank holds the oracle's bits."""
    rng = np.random.default_rng(5000 + seed)
    N = int(rng.integers(2, 17))
    G = int(rng.integers(2, min(N, 6) + 1))
    m = list(range(G)) + [int(v) for v in rng.integers(0, G, N - G)]
    rng.shuffle(m)
    nb = int(rng.integers(1, 5))
    sizes = [int(rng.choice([0, 1, 7, 15, 16, 17, 1000, 8191, 8193, 65537, 300_001])) for _ in range(nb)]
    if seed % 5 == 3:                     # chunks above 2^20 elements: the pipelined CHAIN cuts W >= 2 tiles
        sizes[0] = int(N * (1 << 20) + rng.integers(1, 3 * (1 << 20)))
    sizes[0] = max(sizes[0], 1)                                   # at least one non-empty bucket
    dts = [str(rng.choice(["f32", "bf16"])) for _ in range(nb)]
    A = int(rng.choice([8, 16, 64, 1024]))
    sched = int(rng.choice(list(SCHED_NAMES)))
    options = int(rng.choice([0, es.ES_OPT_PEER_ROUNDS]))
    if seed % 3 == 2:                                             # a third of the seeds push the gather
        options |= es.ES_OPT_PEER_PUSH
    if seed % 4 == 1:                                             # a quarter fold at the stash (NEXT-1)
        options |= es.ES_OPT_INCREMENTAL
    steps = int(rng.integers(1, 4))
    xs = [_gauss(rng, N, L, d) for L, d in zip(sizes, dts)]
    want = [oracle.reduce(x, d, A=A) for x, d in zip(xs, dts)]
    what = f"seed={seed} N={N} G={G} map={m} sizes={sizes} dts={dts} A={A} {SCHED_NAMES[sched]} opt={options}"
    res = reduce_loopback(xs, G, m, sched, A=A, steps=steps, batched=bool(seed % 2), options=options)
    for g in range(G):
        for b in range(nb):
            assert_bits_equal(res[g][b], want[b], f"{what} rank={g} b={b}")


# ---- ES_OPT_STASH_BACKGROUND (one-wave stash / incremental-fold grids) ------------------------

@pytest.mark.parametrize("incremental", [False, True])
def test_stash_background_grid_bit_exact(incremental):
    """The capped switch-time grid changes only which CTA does which element."""
    from gpu_util import Aggregator, from_dev, to_dev
    N = 8
    rng = np.random.default_rng(1300 + incremental)
    Ls, dts = [3_000_017, 40, 77_777], ["f32", "bf16", "f32"]
    opts = es.ES_OPT_STASH_BACKGROUND | (es.ES_OPT_INCREMENTAL if incremental else 0)
    agg = Aggregator(N, 1, 0, [0] * N, list(zip(Ls, dts)), options=opts)
    outs = [agg.new_out(b) for b in range(len(Ls))]
    xs = [_gauss(rng, N, L, d) for L, d in zip(Ls, dts)]
    devs = [[to_dev(xs[b][k]) for b in range(len(Ls))] for k in range(N)]
    for k in range(N):
        mode = es.ES_STASH_BORROW if k == N - 1 else es.ES_STASH_COPY
        if incremental:
            agg.stash_fold(k, range(len(Ls)), devs[k], mode)
        else:
            agg.stash_many(k, range(len(Ls)), devs[k], mode)
    agg.allreduce_many(range(len(Ls)), outs)
    torch.cuda.synchronize()
    for b, d in enumerate(dts):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], d), f"b={b}")
    agg.close()


# ---- small-fold kernel selection (k_fold<F32WT>) ------------------------------------------------

@pytest.mark.parametrize("L", [8, 17, 10007, 1 << 20, (1 << 21) + 16])
def test_small_fold_wide_and_narrow_paths(L):
    """fp32 folds of <= 2^21 elements with 32-byte aligned pointers run 8 elements per thread
    (k_fold<F32WT>); a BORROWed gradient and an output that are only 16-byte aligned take the
    F32T kernel; above 2^21 elements F32T as well.  Every path gives the oracle's bits."""
    from gpu_util import Aggregator, from_dev, to_dev
    N = 4
    rng = np.random.default_rng(2100 + L % 97)
    xs = _gauss(rng, N, L)
    want = oracle.reduce(xs, "f32")
    for offset in (0, 4):                  # 4 floats = 16 bytes: breaks 32-byte alignment only
        agg = Aggregator(N, 1, 0, [0] * N, [(L, "f32")])
        base = [torch.zeros(L + 8, dtype=torch.float32, device="cuda") for _ in range(N)]
        devs = []
        for k in range(N):
            base[k][offset:offset + L].copy_(to_dev(xs[k]))
            devs.append(base[k][offset:offset + L])
        out_base = torch.zeros(L + 8, dtype=torch.float32, device="cuda")
        out = out_base[offset:offset + L]
        for k in range(N):
            agg.stash(k, 0, devs[k], es.ES_STASH_BORROW if k == N - 1 else es.ES_STASH_COPY)
        agg.allreduce(0, out)
        torch.cuda.synchronize()
        assert_bits_equal(from_dev(out), want, f"L={L} offset={offset}")
        agg.close()
