"""CPU: replay libes's actual plan (exported through the C ABI) on the host
for every G and EST->GPU mapping, and require the oracle's bits on every
rank (D1: the result must not depend on the number of GPUs
or on placement).  SURVEY.md 8(c) 'Invariance' pin: all surjective maps for
N=4, G in {1,2,3,4} and N=6, G=3."""
import itertools

import numpy as np
import pytest

import oracle
from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads

from plan_sim import simulate


def _data(N, Ls, dtypes, seed):
    rng = np.random.default_rng(seed)
    xs = []
    for L, d in zip(Ls, dtypes):
        mu = rng.standard_normal(L) * 1e-3
        row = [(mu + rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
        xs.append(row if d == "f32" else [oracle.f32_to_bf16_bits(x) for x in row])
    return xs


def _surjections(N, G):
    for m in itertools.product(range(G), repeat=N):
        if len(set(m)) == G:
            yield list(m)


def _check(N, G, mapping, Ls, dtypes, sched, A=16, seed=0, xs=None, want=None):
    xs = xs or _data(N, Ls, dtypes, seed)
    want = want or [oracle.reduce(x, d, A=A) for x, d in zip(xs, dtypes)]
    ranks = simulate(N, G, mapping, list(zip(Ls, dtypes)), xs, A=A, sched=sched)
    for r in ranks:
        for b, d in enumerate(dtypes):
            got = r.out[b]
            assert np.array_equal(got.view(np.uint32 if d == "f32" else np.uint16),
                                  want[b].view(np.uint32 if d == "f32" else np.uint16)), \
                f"map={mapping} sched={sched} rank={r.g} bucket={b}"
    return ranks


@pytest.mark.parametrize("G", [1, 2, 3, 4])
def test_all_surjections_n4(G):
    Ls, dts = [203, 64, 5, 0], ["f32", "bf16", "f32", "f32"]
    xs = _data(4, Ls, dts, G)
    want = [oracle.reduce(x, d) for x, d in zip(xs, dts)]
    for m in _surjections(4, G):
        for sched in (es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN, es.ES_SCHED_AUTO, es.ES_SCHED_PEER,
                      es.ES_SCHED_PEER_CHAIN, es.ES_SCHED_PEER_AUTO):
            _check(4, G, m, Ls, dts, sched, xs=xs, want=want)


@pytest.mark.slow
def test_all_surjections_n6_g3():
    Ls, dts = [301, 48], ["f32", "bf16"]
    xs = _data(6, Ls, dts, 63)
    want = [oracle.reduce(x, d) for x, d in zip(xs, dts)]
    n = 0
    for m in _surjections(6, 3):
        for sched in (es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN, es.ES_SCHED_PEER, es.ES_SCHED_PEER_CHAIN):
            _check(6, 3, m, Ls, dts, sched, xs=xs, want=want)
        n += 1
    assert n == 540


@pytest.mark.parametrize("name,G,kind", [("resnet50", 2, "contiguous"), ("resnet50", 8, "random"),
                                         ("vgg19", 4, "contiguous"), ("bert_base", 8, "contiguous"),
                                         ("bert_base", 8, "round_robin"), ("swin_b", 8, "contiguous"),
                                         ("swin_b", 2, "round_robin")])
def test_config_shapes_small_buckets(name, G, kind):
    """The paper configs' N, G and mappings, on small ragged buckets."""
    N = workloads.config(name)["N"]
    d = workloads.config(name)["dtype"]
    m = workloads.mapping(N, G, kind)
    for sched in (es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN, es.ES_SCHED_AUTO, es.ES_SCHED_PEER,
                      es.ES_SCHED_PEER_CHAIN, es.ES_SCHED_PEER_AUTO):
        _check(N, G, m, [997, 4096 + 24, 13], [d, d, d], sched, seed=G)


def test_chain_partials_cross_gpus_in_canonical_order():
    """Chain on a contiguous map sends each chunk's partial at most G
    times + the wrap; it never sends raw contributions."""
    N, G = 8, 4
    m = workloads.mapping(N, G, "contiguous")
    for g in range(G):
        ops, sched = es.es_plan_ops(es.Config(N, G, g, m, [(1 << 16, es.ES_F32)], sched=es.ES_SCHED_CHAIN), 0)
        assert sched == es.ES_SCHED_CHAIN
        sends = ops[ops[:, 0] == es.ES_OP_SEND]
        assert set(sends[:, 4].tolist()) <= {es.ES_BUF_PART, es.ES_BUF_OUT}


def test_auto_picks_fewer_bytes():
    """SURVEY.md 8(e) planner rule: chain for fp32 with n_g >= 2 on contiguous
    maps (VGG-19 G=2), direct when n_g = 1 (ResNet-50 G=8)."""
    def sched_of(name, G, kind="contiguous"):
        c = workloads.config(name)
        cfg = es.Config(c["N"], G, 0, workloads.mapping(c["N"], G, kind),
                        [(n, es.ES_F32 if d == "f32" else es.ES_BF16) for n, d in c["buckets"]])
        return es.es_plan_ops(cfg, 1)[1]
    assert sched_of("vgg19", 2) == es.ES_SCHED_CHAIN
    assert sched_of("swin_b", 4) == es.ES_SCHED_CHAIN
    assert sched_of("resnet50", 8) == es.ES_SCHED_DIRECT
    assert sched_of("bert_base", 8, "round_robin") == es.ES_SCHED_DIRECT


def test_random_configs_property():
    """Property test over random (N, G, mapping, ragged L, A, schedule): every
    rank of the replayed plan holds the oracle's bits."""
    from hypothesis import given, settings, HealthCheck
    from hypothesis import strategies as st

    @st.composite
    def cfgs(draw):
        N = draw(st.integers(1, 12))
        G = draw(st.integers(1, min(N, 6)))
        base = list(range(G)) + [draw(st.integers(0, G - 1)) for _ in range(N - G)]
        perm = draw(st.permutations(base))
        nb = draw(st.integers(1, 3))
        Ls = [draw(st.integers(0, 700)) for _ in range(nb)]
        dts = [draw(st.sampled_from(["f32", "bf16"])) for _ in range(nb)]
        A = draw(st.sampled_from([8, 16, 32]))
        sched = draw(st.sampled_from([es.ES_SCHED_AUTO, es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN, es.ES_SCHED_PEER,
                                      es.ES_SCHED_PEER_CHAIN, es.ES_SCHED_PEER_AUTO]))
        seed = draw(st.integers(0, 2 ** 31))
        return N, G, list(perm), Ls, dts, A, sched, seed

    @settings(max_examples=150, deadline=None, suppress_health_check=list(HealthCheck))
    @given(cfgs())
    def run(c):
        N, G, m, Ls, dts, A, sched, seed = c
        xs = _data(N, [max(L, 1) for L in Ls], dts, seed)
        xs = [[x[:L] for x in row] for row, L in zip(xs, Ls)]
        want = [oracle.reduce(x, d, A=A) for x, d in zip(xs, dts)]
        _check(N, G, m, Ls, dts, sched, A=A, xs=xs, want=want)

    run()
