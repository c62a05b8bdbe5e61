"""GPU: D2 analogue on B200 -- the aggregation run inside CUDA green contexts
restricted to a few SMs gives the same bits as on the whole GPU.

PAPER.md:774-780 (D2) pins reduce kernels to "a specific number of SMs and
threads" so that results do not depend on the GPU.  Here the opposite
direction is tested: the canonical fold and the stash are run on SM
partitions of 8, 16 and 32 SMs (cuGreenCtxCreate over a
cuDevSmResourceSplitByCount group) and must match the oracle bit for bit
-- the kernels' results never depend on how many SMs execute them.
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_lixyszrljlllq23_b200 import es
from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator

from gpu_util import assert_bits_equal, from_dev, to_dev

pytestmark = pytest.mark.gpu


def _check(res):
    err = res[0]
    if int(err) != 0:
        raise RuntimeError(f"driver error {err}")
    return res[1:] if len(res) > 2 else (res[1] if len(res) == 2 else None)


def _green_stream(n_sms):
    from cuda.bindings import driver as cu
    dev = _check(cu.cuDeviceGet(torch.cuda.current_device()))
    res = _check(cu.cuDeviceGetDevResource(dev, cu.CUdevResourceType.CU_DEV_RESOURCE_TYPE_SM))
    groups, nb, remaining = _check(cu.cuDevSmResourceSplitByCount(1, res, 0, n_sms))
    desc = _check(cu.cuDevResourceGenerateDesc([groups[0]], 1))
    gctx = _check(cu.cuGreenCtxCreate(desc, dev, cu.CUgreenCtxCreate_flags.CU_GREEN_CTX_DEFAULT_STREAM))
    stream = _check(cu.cuGreenCtxStreamCreate(gctx, cu.CUstream_flags.CU_STREAM_NON_BLOCKING, 0))
    ctx = _check(cu.cuCtxFromGreenCtx(gctx))
    return cu, gctx, ctx, stream, groups[0].sm.smCount


@pytest.mark.parametrize("n_sms", [8, 16, 32])
def test_fold_on_green_context_sm_partitions(n_sms):
    torch.cuda.init()
    try:
        cu, gctx, ctx, stream, got_sms = _green_stream(n_sms)
    except Exception as e:  # green contexts unavailable on this driver / device
        pytest.skip(f"green contexts unavailable: {e}")
    rng = np.random.default_rng(n_sms)
    N, Ls, dts = 8, [300007, 4099, 17], ["f32", "bf16", "f32"]
    xs = []
    for L, d in zip(Ls, dts):
        row = [(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
        xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
    devs = [[to_dev(xs[b][k]) for b in range(3)] for k in range(N)]
    agg = Aggregator(N, 1, 0, [0] * N, list(zip(Ls, dts)))
    outs = [agg.new_out(b) for b in range(3)]
    torch.cuda.synchronize()
    _check(cu.cuCtxPushCurrent(ctx))
    try:
        s = int(stream)
        for k in range(N):
            es.es_stash_grads(agg.h, k, list(range(3)), [devs[k][b].data_ptr() for b in range(3)],
                              [es.ES_F32 if d == "f32" else es.ES_BF16 for d in dts],
                              es.ES_STASH_BORROW if k == N - 1 else es.ES_STASH_COPY, s)
        es.es_allreduce_many(agg.h, list(range(3)), [o.data_ptr() for o in outs], s)
        _check(cu.cuStreamSynchronize(stream))
    finally:
        _check(cu.cuCtxPopCurrent())
    for b, d in enumerate(dts):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], d), f"{got_sms} SMs, bucket {b}")
    agg.close()
    cu.cuStreamDestroy(stream)
    cu.cuGreenCtxDestroy(gctx)


def test_green_context_really_restricts_sms():
    """Evidence that the partition applies: the same fold on 8 SMs is several
    times slower than on the whole GPU, and still bit-identical."""
    import time
    torch.cuda.init()
    try:
        cu, gctx, ctx, stream, got_sms = _green_stream(8)
    except Exception as e:
        pytest.skip(f"green contexts unavailable: {e}")
    N, L = 8, 1 << 25
    g = torch.Generator(device="cuda").manual_seed(8)
    xs = [torch.randn(L, generator=g, device="cuda") * 1e-3 for _ in range(N)]
    agg = Aggregator(N, 1, 0, [0] * N, [(L, "f32")])
    out_full, out_green = agg.new_out(0), agg.new_out(0)

    def run(out, s):
        for k in range(N):
            es.es_stash_grad(agg.h, k, 0, xs[k].data_ptr(), es.ES_F32, es.ES_STASH_BORROW, s)
        es.es_allreduce(agg.h, 0, out.data_ptr(), s)

    def timed(fn, sync):
        fn()
        sync()
        t0 = time.perf_counter()
        for _ in range(5):
            fn()
        sync()
        return (time.perf_counter() - t0) / 5

    t_full = timed(lambda: run(out_full, torch.cuda.current_stream().cuda_stream), torch.cuda.synchronize)
    _check(cu.cuCtxPushCurrent(ctx))
    try:
        t_green = timed(lambda: run(out_green, int(stream)), lambda: _check(cu.cuStreamSynchronize(stream)))
    finally:
        _check(cu.cuCtxPopCurrent())
    assert torch.equal(out_full.view(torch.int32), out_green.view(torch.int32))
    assert t_green > 3 * t_full, (t_green, t_full, got_sms)
    agg.close()
    cu.cuStreamDestroy(stream)
    cu.cuGreenCtxDestroy(gctx)


@pytest.mark.parametrize("n_sms", [8, 16, 32])
def test_dropout_on_green_context_sm_partitions(n_sms):
    """NEXT-4 (D2): the per-EST dropout, driven by each EST's
    swapped device Philox record, gives the oracle's masks and values on an SM
    partition of 8/16/32 SMs -- time-sliced ESTs, switches on the same green
    stream, several calls per EST (the offset advances once per call)."""
    torch.cuda.init()
    try:
        cu, gctx, ctx, stream, got_sms = _green_stream(n_sms)
    except Exception as e:  # green contexts unavailable on this driver / device
        pytest.skip(f"green contexts unavailable: {e}")
    N, calls, p = 4, 2, 0.3
    seeds = [0x5EED_0000_0000 + 977 * k for k in range(N)]
    rng = np.random.default_rng(100 + n_sms)
    sizes = {"f32": 300007, "bf16": 4099}
    xs = {}
    for d, n in sizes.items():
        x32 = rng.standard_normal(n).astype(np.float32)
        xs[d] = x32 if d == "f32" else oracle.f32_to_bf16_bits(x32)
    agg = Aggregator(N, 1, 0, [0] * N, [(64, "f32")], state_nbytes=[16])
    live = [torch.zeros(16, dtype=torch.uint8, device="cuda")]
    agg.register_state(live)
    for k in range(N):
        agg.init_state(k, 0, int(seeds[k]).to_bytes(8, "little") + (0).to_bytes(8, "little"))
    xdev = {d: to_dev(x) for d, x in xs.items()}
    ys = {(k, c, d): torch.empty_like(xdev[d]) for k in range(N) for c in range(calls) for d in sizes}
    ms = {(k, c, d): torch.empty(sizes[d], dtype=torch.uint8, device="cuda")
          for k in range(N) for c in range(calls) for d in sizes}
    torch.cuda.synchronize()
    _check(cu.cuCtxPushCurrent(ctx))
    try:
        s = int(stream)
        for k in range(N):
            es.es_switch_context(agg.h, k, s)
            for c in range(calls):
                for d in sizes:
                    es.es_dropout(agg.h, xdev[d].data_ptr(), ys[(k, c, d)].data_ptr(), ms[(k, c, d)].data_ptr(),
                                  sizes[d], es.ES_F32 if d == "f32" else es.ES_BF16, p, 0, s)
        _check(cu.cuStreamSynchronize(stream))
    finally:
        _check(cu.cuCtxPopCurrent())
    for k in range(N):
        off = 0
        for c in range(calls):
            for d in sizes:                       # one offset unit per es_dropout call, in call order
                wy, wm = oracle.dropout(xs[d], d, p, seeds[k], off)
                assert np.array_equal(ms[(k, c, d)].cpu().numpy(), wm), (got_sms, k, c, d)
                assert_bits_equal(from_dev(ys[(k, c, d)]), wy, f"{got_sms} SMs, EST {k} call {c} {d}")
                off += 1
    agg.close()
    cu.cuStreamDestroy(stream)
    cu.cuGreenCtxDestroy(gctx)
