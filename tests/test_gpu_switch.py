"""GPU: context switch (k_swap) and the C-ABI protocol errors.

PAPER.md:575-598 -- an EST's context is its RNG state and implicit per-worker
state such as BatchNorm running statistics; only that (plus the
gradients) is swapped at a mini-batch boundary.  The oracle is
oracle/switch_model.py: after any interleaving of switches and updates,
every EST's state equals what a dedicated worker would hold."""
import numpy as np
import pytest
import torch

from oracle.switch_model import SwitchModel
from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads
from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator

pytestmark = pytest.mark.gpu

SIZES = [16, workloads.BN_F32 * 4, workloads.BN_I64 * 8, 37]   # Philox record, BN stats, counters, ragged


def _setup(N, seed):
    rng = np.random.default_rng(seed)
    agg = Aggregator(N, 1, 0, [0] * N, [(64, "f32")], state_nbytes=SIZES)
    live = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in SIZES]
    agg.register_state(live)
    init = {k: [rng.integers(0, 256, n, dtype=np.uint8).tobytes() for n in SIZES] for k in range(N)}
    for k in range(N):
        for i in range(len(SIZES)):
            agg.init_state(k, i, init[k][i])
    return agg, live, init, rng


def _live_bytes(live):
    torch.cuda.synchronize()
    return [t.cpu().numpy().tobytes() for t in live]


@pytest.mark.parametrize("N", [1, 4, 32])
def test_switch_model_random_sequences(N):
    agg, live, init, rng = _setup(N, N)
    model = SwitchModel(N, init)
    agg.switch(0)                       # first switch only loads
    assert _live_bytes(live) == model.state_of(0)
    cur = 0
    for step in range(200):
        if rng.random() < 0.4:          # the running EST updates its context (BN update, RNG advance)
            i = int(rng.integers(0, len(SIZES)))
            nb = rng.integers(0, 256, SIZES[i], dtype=np.uint8)
            live[i].copy_(torch.from_numpy(nb).cuda())
            model.mutate(i, nb.tobytes())
        else:
            k = int(rng.integers(0, N))
            agg.switch(k)
            model.switch(k)
            cur = k
        if step % 10 == 0:
            assert _live_bytes(live) == model.state_of(cur)
            torch.cuda.synchronize()
            for k in range(N):
                if k != cur:
                    assert [agg.read_state(k, i) for i in range(len(SIZES))] == model.state_of(k)
    agg.sync()
    agg.close()


def test_switch_to_self_is_identity_and_round_trip():
    agg, live, init, _ = _setup(3, 1)
    agg.switch(1)
    before = _live_bytes(live)
    agg.switch(1)
    assert _live_bytes(live) == before
    agg.switch(2)
    agg.switch(1)
    assert _live_bytes(live) == before      # round trip restores the bits
    agg.close()


def test_dropout_masks_follow_the_est():
    """R12: an EST's dropout masks under time-slicing equal those of a dedicated
    worker seeded the same way (D0 fixed seeds)."""
    N, steps = 4, 3
    seeds = [1234 + 17 * k for k in range(N)]
    gen = torch.cuda.default_generators[torch.cuda.current_device()]
    x = torch.ones(4096, device="cuda")
    dedicated = {}
    for k in range(N):
        gen.manual_seed(seeds[k])
        dedicated[k] = [torch.nn.functional.dropout(x, 0.5).clone() for _ in range(steps)]
    agg = Aggregator(N, 1, 0, [0] * N, [(64, "f32")])
    agg.attach_generator(gen, seeds)
    for s in range(steps):
        for k in range(N):
            agg.switch(k)
            m = torch.nn.functional.dropout(x, 0.5)
            assert torch.equal(m, dedicated[k][s]), (s, k)
    agg.close()


def test_protocol_errors():
    N = 4
    agg = Aggregator(N, 2, 0, [0, 0, 1, 1], [(1000, "f32")], transport=es.ES_TRANSPORT_LOOPBACK,
                     comm=es.es_loopback_create(2).value)
    g = torch.zeros(1000, device="cuda")
    out = torch.zeros(1000, device="cuda")
    with pytest.raises(es.EsError) as e:
        agg.stash(2, 0, g)                              # EST 2 lives on rank 1
    assert e.value.status == es.ES_ESTATE
    with pytest.raises(es.EsError) as e:
        agg.stash(9, 0, g)
    assert e.value.status == es.ES_EINVAL
    with pytest.raises(es.EsError) as e:
        agg.stash(0, 3, g)
    assert e.value.status == es.ES_EINVAL
    with pytest.raises(es.EsError) as e:
        es.es_stash_grad(agg.h, 0, 0, g.data_ptr() + 4, es.ES_F32, es.ES_STASH_COPY, 0)   # misaligned
    assert e.value.status == es.ES_EINVAL
    with pytest.raises(es.EsError) as e:
        agg.stash(0, 0, g.to(torch.bfloat16), es.ES_STASH_BORROW)   # borrow needs the bucket dtype
    assert e.value.status == es.ES_EINVAL
    agg.stash(0, 0, g)
    with pytest.raises(es.EsError) as e:
        agg.allreduce(0, out)                           # EST 1 has not stashed
    assert e.value.status == es.ES_ESTATE
    with pytest.raises(es.EsError) as e:
        agg.switch(3)
    assert e.value.status == es.ES_ESTATE
    with pytest.raises(es.EsError) as e:
        es.es_allreduce(agg.h, 0, agg.workspace.data_ptr() + 256, 0)   # out inside the workspace
    assert e.value.status == es.ES_EINVAL
    agg.close()


def test_init_errors():
    cfg = es.Config(4, 1, 0, [0] * 4, [(100, es.ES_F32)])
    nb = es.es_workspace_bytes(cfg)
    ws = torch.empty(nb + 512, dtype=torch.uint8, device="cuda")
    with pytest.raises(es.EsError) as e:
        es.es_init(cfg, ws.data_ptr(), nb - 256)
    assert e.value.status == es.ES_ENOMEM
    with pytest.raises(es.EsError) as e:
        es.es_init(cfg, ws.data_ptr() + 16, nb)
    assert e.value.status == es.ES_EINVAL
    host = torch.empty(nb + 256, dtype=torch.uint8)
    ptr = (host.data_ptr() + 255) // 256 * 256
    with pytest.raises(es.EsError) as e:
        es.es_init(cfg, ptr, nb)
    assert e.value.status == es.ES_EINVAL
    h = es.es_init(cfg, ws.data_ptr(), nb)
    es.es_destroy(h)


def test_stash_and_switch_fused():
    """es_stash_and_switch == es_stash_grads + es_switch_context: same fold
    bits (oracle) and same per-EST context (switch model), one launch each."""
    import oracle
    from gpu_util import assert_bits_equal, from_dev, to_dev
    N = 6
    rng = np.random.default_rng(21)
    Ls = [70001, 33, 4096]
    xs = [[(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)] for L in Ls]
    agg = Aggregator(N, 1, 0, [0] * N, [(L, "f32") for L in Ls], state_nbytes=SIZES)
    live = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in SIZES]
    agg.register_state(live)
    init = {k: [rng.integers(0, 256, n, dtype=np.uint8).tobytes() for n in SIZES] for k in range(N)}
    for k in range(N):
        for i in range(len(SIZES)):
            agg.init_state(k, i, init[k][i])
    model = SwitchModel(N, init)
    devs = [[to_dev(xs[b][k]) for b in range(len(Ls))] for k in range(N)]
    outs = [agg.new_out(b) for b in range(len(Ls))]
    for step in range(3):
        agg.switch(0)
        model.switch(0)
        for k in range(N):
            nb = rng.integers(0, 256, SIZES[1], dtype=np.uint8)   # EST k's local step updates its BN stats
            live[1].copy_(torch.from_numpy(nb).cuda())
            model.mutate(1, nb.tobytes())
            agg.profile(True)
            agg.profile_reset()
            if k < N - 1:
                agg.stash_and_switch(k, range(len(Ls)), devs[k], k + 1)
                model.switch(k + 1)
                n_st, _, _ = agg.profile_query(es.ES_KERNEL_STASH)
                n_sw, _, _ = agg.profile_query(es.ES_KERNEL_SWAP)
                assert (n_st, n_sw) == (1, 0)          # one fused launch
            else:
                agg.stash_many(k, range(len(Ls)), devs[k], es.ES_STASH_BORROW)
            agg.profile(False)
            torch.cuda.synchronize()
            assert _live_bytes(live) == model.state_of(k + 1 if k < N - 1 else k)
        agg.allreduce_many(range(len(Ls)), outs)
        torch.cuda.synchronize()
        for b in range(len(Ls)):
            assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], "f32"), f"step {step} b={b}")
        for k in range(N - 1):
            assert [agg.read_state(k, i) for i in range(len(SIZES))] == model.state_of(k)
    agg.close()


# ---- NEXT-2: zero-copy stash and elastic resume --------------------------------------------

def test_inplace_stash_moves_no_bytes():
    import oracle
    from gpu_util import assert_bits_equal, from_dev
    N, Ls = 5, [40001, 1000, 7]
    rng = np.random.default_rng(31)
    xs = [[(rng.standard_normal(L) * 1e-2).astype(np.float32) for _ in range(N)] for L in Ls]
    agg = Aggregator(N, 1, 0, [0] * N, [(L, "f32") for L in Ls])
    for k in range(N):
        for b in range(len(Ls)):
            agg.slot(k, b).copy_(torch.from_numpy(xs[b][k]).cuda())   # "backward" writes into the slot
    agg.profile(True)
    agg.profile_reset()
    for k in range(N):
        agg.stash_many(k, range(len(Ls)), [agg.slot(k, b) for b in range(len(Ls))], es.ES_STASH_INPLACE)
    assert agg.profile_query(es.ES_KERNEL_STASH)[0] == 0
    outs = [agg.new_out(b) for b in range(len(Ls))]
    agg.allreduce_many(range(len(Ls)), outs)
    torch.cuda.synchronize()
    for b in range(len(Ls)):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], "f32"))
    with pytest.raises(es.EsError) as e:       # INPLACE must name the slot itself
        agg.stash(0, 0, torch.zeros(Ls[0], device="cuda"), es.ES_STASH_INPLACE)
    assert e.value.status == es.ES_EINVAL
    agg.close()


def _threads(G, fn):
    import threading
    errs = []
    dev = torch.cuda.current_device()

    def run(g):
        try:
            torch.cuda.set_device(dev)
            fn(g)
        except Exception as ex:
            errs.append(ex)
    ts = [threading.Thread(target=run, args=(g,)) for g in range(G)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout=300)
    torch.cuda.synchronize()
    if errs:
        raise errs[0]


def test_elastic_resume_mid_step_fig9():
    """Synthetic Fig. 9: a global step starts on G=4, is
    revoked after 5 of 8 ESTs ran (on-demand checkpoint of every EST context,
    P:608-624), resumes on G=2 with another mapping, and the next step runs on
    G=3 unevenly.  Every aggregate equals the oracle (and hence G=1) bit for
    bit, and every EST's context continues unchanged (D1)."""
    import oracle
    from gpu_util import assert_bits_equal, from_dev, to_dev
    from paper_conf_sc_lixyszrljlllq23_b200 import workloads as wl
    N, Ls, dts = 8, [30011, 4096, 9], ["f32", "bf16", "f32"]
    rng = np.random.default_rng(41)

    def data():
        out = []
        for L, d in zip(Ls, dts):
            row = [(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
            out.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
        return out

    init = {k: [rng.integers(0, 256, n, dtype=np.uint8).tobytes() for n in SIZES] for k in range(N)}

    def stage(G, mapping):
        world = es.es_loopback_create(G)
        aggs = [Aggregator(N, G, g, mapping, list(zip(Ls, dts)), state_nbytes=SIZES,
                           transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value) for g in range(G)]
        lives = []
        for a in aggs:
            live = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in SIZES]
            a.register_state(live)
            lives.append(live)
        return world, aggs, lives

    def allreduce(G, aggs):
        outs = [[a.new_out(b) for b in range(len(Ls))] for a in aggs]
        streams = [torch.cuda.Stream() for _ in range(G)]
        torch.cuda.synchronize()

        def fn(g):
            with torch.cuda.stream(streams[g]):
                aggs[g].allreduce_many(range(len(Ls)), outs[g])
        _threads(G, fn)
        return outs

    def check(outs, xs, what):
        for g, row in enumerate(outs):
            for b in range(len(Ls)):
                assert_bits_equal(from_dev(row[b]), oracle.reduce(xs[b], dts[b]), f"{what} rank {g} bucket {b}")

    # stage 0: G=4 contiguous; one full step
    m0 = wl.mapping(N, 4, "contiguous")
    w0, aggs0, _ = stage(4, m0)
    for k in range(N):
        for i in range(len(SIZES)):
            aggs0[m0[k]].init_state(k, i, init[k][i])
    x1 = data()
    d1 = [[to_dev(x1[b][k]) for b in range(len(Ls))] for k in range(N)]
    for k in range(N):
        aggs0[m0[k]].stash_many(k, range(len(Ls)), d1[k])
    check(allreduce(4, aggs0), x1, "stage0 step1")
    # step 2 starts: ESTs 0..4 run (stash), then the job is revoked
    x2 = data()
    d2 = [[to_dev(x2[b][k]) for b in range(len(Ls))] for k in range(N)]
    for k in range(5):
        aggs0[m0[k]].stash_many(k, range(len(Ls)), d2[k],
                                es.ES_STASH_BORROW if k == 4 else es.ES_STASH_COPY)
    torch.cuda.synchronize()
    blobs = {k: aggs0[m0[k]].export_context(k) for k in range(N)}
    for a in aggs0:
        a.close()
    es.es_loopback_destroy(w0)

    # stage 1: G=2 round robin; resume mid-step
    m1 = wl.mapping(N, 2, "round_robin")
    w1, aggs1, _ = stage(2, m1)
    for k in range(N):
        aggs1[m1[k]].import_context(k, blobs[k])
    for k in range(5, N):
        aggs1[m1[k]].stash_many(k, range(len(Ls)), d2[k])
    check(allreduce(2, aggs1), x2, "stage1 resumed step2")
    for k in range(N):                               # contexts survived the move
        assert [aggs1[m1[k]].read_state(k, i) for i in range(len(SIZES))] == init[k]
    blobs = {k: aggs1[m1[k]].export_context(k) for k in range(N)}
    for a in aggs1:
        a.close()
    es.es_loopback_destroy(w1)

    # stage 2: G=3 uneven random mapping; a fresh step
    m2 = wl.mapping(N, 3, "random", seed=3)
    w2, aggs2, _ = stage(3, m2)
    for k in range(N):
        aggs2[m2[k]].import_context(k, blobs[k])
    x3 = data()
    d3 = [[to_dev(x3[b][k]) for b in range(len(Ls))] for k in range(N)]
    for k in range(N):
        aggs2[m2[k]].stash_many(k, range(len(Ls)), d3[k])
    check(allreduce(3, aggs2), x3, "stage2 step3")
    # a layout change is refused (D0 failure mode)
    other = Aggregator(N, 1, 0, [0] * N, [(L + 16, d) for L, d in zip(Ls, dts)], state_nbytes=SIZES)
    with pytest.raises(es.EsError) as e:
        other.import_context(0, blobs[0])
    assert e.value.status == es.ES_ESTATE
    other.close()
    for a in aggs2:
        a.close()
    es.es_loopback_destroy(w2)


# ---- NEXT-4: per-EST device Philox dropout --------------------------------------------------

def _philox_state(seed, offset=0):
    return int(seed).to_bytes(8, "little") + int(offset).to_bytes(8, "little")


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_dropout_matches_oracle(dtype):
    import oracle
    from gpu_util import assert_bits_equal, from_dev, to_dev
    agg = Aggregator(1, 1, 0, [0], [(64, "f32")], state_nbytes=[16])
    live = [torch.zeros(16, dtype=torch.uint8, device="cuda")]
    agg.register_state(live)
    seed, off = 0x1234_5678_9ABC_DEF0, 41
    agg.init_state(0, 0, _philox_state(seed, off))
    agg.switch(0)
    rng = np.random.default_rng(7)
    for n, p in [(1, 0.5), (5, 0.1), (4099, 0.5), (100003, 0.9), (65536, 0.0)]:
        x32 = rng.standard_normal(n).astype(np.float32)
        x = x32 if dtype == "f32" else oracle.f32_to_bf16_bits(x32)
        y, m = agg.dropout(to_dev(x), p, with_mask=True)
        torch.cuda.synchronize()
        wy, wm = oracle.dropout(x, dtype, p, seed, off)
        assert np.array_equal(m.cpu().numpy(), wm), (n, p)
        assert_bits_equal(from_dev(y), wy, f"n={n} p={p}")
        off += 1                                                  # one offset unit per call
        assert live[0].cpu().numpy().tobytes() == _philox_state(seed, off)
    agg.close()


def _dedicated_masks(seeds, steps, calls, n, p):
    out = {}
    for k, seed in enumerate(seeds):
        a = Aggregator(1, 1, 0, [0], [(64, "f32")], state_nbytes=[16])
        live = [torch.zeros(16, dtype=torch.uint8, device="cuda")]
        a.register_state(live)
        a.init_state(0, 0, _philox_state(seed))
        a.switch(0)
        x = torch.ones(n, device="cuda")
        out[k] = [[a.dropout(x, p, with_mask=True)[1].clone() for _ in range(calls)] for _ in range(steps)]
        torch.cuda.synchronize()
        a.close()
    return out


def test_dropout_time_sliced_equals_dedicated_and_graph_safe():
    """An EST's masks do not depend on how ESTs share a GPU -- eager and inside
    a CUDA graph (where a host-side generator mirror could not follow)."""
    N, steps, calls, n, p = 4, 3, 2, 20000, 0.3
    seeds = [1000 + 7 * k for k in range(N)]
    want = _dedicated_masks(seeds, steps, calls, n, p)
    for use_graph in (False, True):
        agg = Aggregator(N, 1, 0, [0] * N, [(64, "f32")], state_nbytes=[16])
        live = [torch.zeros(16, dtype=torch.uint8, device="cuda")]
        agg.register_state(live)
        for k in range(N):
            agg.init_state(k, 0, _philox_state(seeds[k]))
        x = torch.ones(n, device="cuda")
        masks = [[torch.empty(n, dtype=torch.uint8, device="cuda") for _ in range(calls)] for _ in range(N)]

        def one_step():
            for k in range(N):
                agg.switch(k)
                for c in range(calls):
                    es.es_dropout(agg.h, x.data_ptr(), ybuf.data_ptr(),
                                  masks[k][c].data_ptr(), n, es.ES_F32, p, 0, torch.cuda.current_stream().cuda_stream)
        ybuf = torch.empty_like(x)
        if use_graph:
            s = torch.cuda.Stream()
            g = torch.cuda.CUDAGraph()
            agg.switch(N - 1)                      # the step starts with EST N-1 live, as after a step
            torch.cuda.synchronize()
            # capture consumes nothing: records only advance when the graph runs
            with torch.cuda.graph(g, stream=s):
                one_step()
        for st in range(steps):
            if use_graph:
                g.replay()
            else:
                one_step()
            torch.cuda.synchronize()
            for k in range(N):
                for c in range(calls):
                    assert torch.equal(masks[k][c], want[k][st][c]), (use_graph, st, k, c)
        agg.close()
