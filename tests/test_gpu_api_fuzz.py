"""GPU: the C ABI under random misuse.  include/es.h promises that argument
errors (ES_EINVAL) and protocol errors (ES_ESTATE) are detected
synchronously and have no side effects.  A random mix of invalid calls is
interleaved with one valid global step; every invalid call must fail with
the documented status and the step's result must still equal the oracle."""
import ctypes

import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_lixyszrljlllq23_b200 import es
from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator

from gpu_util import assert_bits_equal, from_dev, to_dev

pytestmark = pytest.mark.gpu


def _bad_calls(agg, devs, outs, N, B, rng):
    """Yield (callable, expected status) pairs of invalid calls."""
    L = es.lib()
    h = agg.h
    s = torch.cuda.current_stream().cuda_stream
    g0 = devs[0][0]
    P = ctypes.c_void_p
    cands = [
        (lambda: L.es_stash_grad(h, N, 0, P(g0.data_ptr()), 0, 0, P(s)), es.ES_EINVAL),          # est out of range
        (lambda: L.es_stash_grad(h, -1, 0, P(g0.data_ptr()), 0, 0, P(s)), es.ES_EINVAL),
        (lambda: L.es_stash_grad(h, 0, B, P(g0.data_ptr()), 0, 0, P(s)), es.ES_EINVAL),          # bucket out of range
        (lambda: L.es_stash_grad(h, 0, 0, P(g0.data_ptr() + 4), 0, 0, P(s)), es.ES_EINVAL),      # misaligned
        (lambda: L.es_stash_grad(h, 0, 0, None, 0, 0, P(s)), es.ES_EINVAL),                      # NULL grad
        (lambda: L.es_stash_grad(h, 0, 0, P(g0.data_ptr()), 7, 0, P(s)), es.ES_EINVAL),          # bad dtype
        (lambda: L.es_stash_grad(h, 0, 0, P(g0.data_ptr()), 0, 9, P(s)), es.ES_EINVAL),          # bad mode
        (lambda: L.es_stash_grad(h, 0, 0, P(g0.data_ptr()), 1, 1, P(s)), es.ES_EINVAL),          # BORROW dtype mismatch
        (lambda: L.es_stash_grad(h, 0, 0, P(g0.data_ptr()), 0, 2, P(s)), es.ES_EINVAL),          # INPLACE not the slot
        (lambda: L.es_allreduce(h, B, P(outs[0].data_ptr()), P(s)), es.ES_EINVAL),
        (lambda: L.es_allreduce(h, 0, P(outs[0].data_ptr() + 8), P(s)), es.ES_EINVAL),           # misaligned out
        (lambda: L.es_allreduce(h, 0, P(agg.workspace.data_ptr() + 512), P(s)), es.ES_EINVAL),   # out in workspace
        (lambda: L.es_switch_context(h, N + 3, P(s)), es.ES_EINVAL),
        (lambda: L.es_init_state(h, 0, 5, P(1)), es.ES_EINVAL),                                  # no such state
        (lambda: L.es_dropout(h, P(g0.data_ptr()), P(g0.data_ptr()), None, 16, 0, ctypes.c_float(1.5), 0, P(s)),
         es.ES_EINVAL),                                                                           # p out of range
        (lambda: L.es_set_launch_override(h, 1, 33), es.ES_EINVAL),
        (lambda: L.es_profile_query(h, 99, None, None, None), es.ES_EINVAL),
    ]
    for _ in range(60):
        yield cands[int(rng.integers(0, len(cands)))]


def test_invalid_calls_have_no_side_effects():
    rng = np.random.default_rng(2024)
    N, Ls, dts = 5, [30011, 64, 7], ["f32", "bf16", "f32"]
    xs = []
    for L, d in zip(Ls, dts):
        row = [(rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
        xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
    agg = Aggregator(N, 1, 0, [0] * N, list(zip(Ls, dts)), state_nbytes=[16])
    live = [torch.zeros(16, dtype=torch.uint8, device="cuda")]
    agg.register_state(live)
    for k in range(N):
        agg.init_state(k, 0, bytes(range(16)))
    devs = [[to_dev(xs[b][k]) for b in range(3)] for k in range(N)]
    outs = [agg.new_out(b) for b in range(3)]
    bad = _bad_calls(agg, devs, outs, N, 3, rng)
    agg.switch(0)
    for k in range(N):
        for _ in range(int(rng.integers(0, 4))):              # misuse between the valid calls
            fn, want = next(bad)
            assert fn() == want
        with pytest.raises(es.EsError) as e:                  # protocol: allreduce before all ESTs stashed
            agg.allreduce_many(range(3), outs)
        assert e.value.status == es.ES_ESTATE
        if k == N - 1:
            agg.stash_many(k, range(3), devs[k], es.ES_STASH_BORROW)
        else:
            agg.stash_and_switch(k, range(3), devs[k], k + 1)
    for _ in range(10):
        fn, want = next(bad)
        assert fn() == want
    agg.allreduce_many(range(3), outs)
    torch.cuda.synchronize()
    agg.sync()                                               # no sticky error was left behind
    for b, d in enumerate(dts):
        assert_bits_equal(from_dev(outs[b]), oracle.reduce(xs[b], d), f"bucket {b}")
    agg.close()
