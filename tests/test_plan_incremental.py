"""CPU: the NEXT-1 incremental prefixes the planner exports (es_plan_incremental,
host-only), checked against the rule es.h states for es_stash_fold_grads, for
every surjective EST->GPU map of small N and every schedule, plus a NumPy
replay showing that folding each exported prefix first and continuing over
the rest of the canonical sequence gives the oracle's bits (segmentability,
R14).  SURVEY 8(f) NEXT-1."""
import itertools

import numpy as np
import pytest

import oracle
from paper_conf_sc_lixyszrljlllq23_b200 import es

SCHEDS = [es.ES_SCHED_AUTO, es.ES_SCHED_DIRECT, es.ES_SCHED_CHAIN, es.ES_SCHED_PEER, es.ES_SCHED_PEER_CHAIN,
          es.ES_SCHED_PEER_AUTO]


def _surjections(N, G):
    for m in itertools.product(range(G), repeat=N):
        if len(set(m)) == G:
            yield list(m)


def _chunk(L, N, A=16):
    per = -(-L // N)
    return -(-per // A) * A


def _shard(L, G, h, A=16):
    S = _chunk(L, G, A)
    return min(L, S * h), min(L, S * (h + 1))


def _rows(N, G, rank, m, L, sched, esz=4):
    cfg = es.Config(N, G, rank, m, [(L, es.ES_F32 if esz == 4 else es.ES_BF16)], sched=sched,
                    options=es.ES_OPT_INCREMENTAL)
    ops, sch = es.es_plan_ops(cfg, 0)
    return es.es_plan_incremental(cfg, 0), sch


def _check_rank(N, G, g, m, L, sched, esz=4):
    rows, sch = _rows(N, G, g, m, L, sched, esz)
    C = _chunk(L, N)
    local = [e for e in range(N) if m[e] == g]
    last_local = local[-1]
    seen, seen_q = set(), {}
    for c, first, q, lo, hi in rows.tolist():
        assert c not in seen and (not seen or c > max(seen)), "rows ascend in c"
        seen.add(c)
        assert first == (c + 1) % N and q * esz > 4, "a prefix must save more than the partial costs"
        pre = list(range(first, first + q))
        assert pre[-1] <= N - 1, "the prefix never wraps N-1 -> 0"
        assert all(m[e] == g for e in pre) and last_local not in pre
        clo, chi = min(L, c * C), min(L, (c + 1) * C)
        if sch in (es.ES_SCHED_DIRECT, es.ES_SCHED_PEER):
            slo, shi = _shard(L, G, g)
            assert (lo, hi) == (max(clo, slo), min(chi, shi))
        else:
            assert (lo, hi) == (clo, chi)
        assert hi > lo
        # the run of same-GPU ESTs this rank folds from `first` (chain: its first segment)
        run = 0
        while run < N and m[(first + run) % N] == g:
            run += 1
        seg_len = run if sch in (es.ES_SCHED_CHAIN, es.ES_SCHED_PEER_CHAIN) else N
        assert q <= seg_len - 1, "the end fold keeps at least one source"
        nxt = first + q        # maximal: the prefix stops only where the rule says
        assert nxt >= N or m[nxt] != g or nxt == last_local or q == seg_len - 1
        seen_q[c] = q
    # completeness: every chunk whose sequence starts here with a foldable EST has a row
    for c in range(N):
        first = (c + 1) % N
        clo, chi = min(L, c * C), min(L, (c + 1) * C)
        if sch in (es.ES_SCHED_DIRECT, es.ES_SCHED_PEER):
            slo, shi = _shard(L, G, g)
            clo, chi = max(clo, slo), min(chi, shi)
        run = 0
        while run < N and m[(first + run) % N] == g:
            run += 1
        seg_len = run if sch in (es.ES_SCHED_CHAIN, es.ES_SCHED_PEER_CHAIN) else N
        q = 0                  # the rule, restated: local, ascending, not the last local EST
        while q < seg_len - 1 and first + q < N and m[first + q] == g and first + q != last_local:
            q += 1
        can = m[first] == g and chi > clo and q * esz > 4
        assert (c in seen) == can, f"chunk {c}"
        if can:
            assert seen_q[c] == q
    return rows


@pytest.mark.parametrize("esz", [4, 2])
@pytest.mark.parametrize("N,G", [(4, 1), (4, 2), (4, 3), (4, 4), (6, 3), (5, 2)])
def test_incremental_prefixes_follow_the_rule(N, G, esz):
    for sched in (SCHEDS if G > 1 else [es.ES_SCHED_AUTO]):
        for m in _surjections(N, G):
            for L in (N * 16 * 3 + 5, 40):        # ragged tail; 40 < N*C leaves chunks empty
                owners = {}
                for g in range(G):
                    for c, first, q, lo, hi in _check_rank(N, G, g, m, L, sched, esz).tolist():
                        for i in range(lo, hi):   # every element's partial belongs to one rank
                            assert i not in owners
                            owners[i] = g


def _fold(xs, order, i):
    s = np.float32(xs[order[0]][i])
    for e in order[1:]:
        s = np.float32(s + xs[e][i])
    return s


@pytest.mark.parametrize("N,G,kind", [(8, 2, "contiguous"), (8, 4, "contiguous"), (8, 3, "random"),
                                      (12, 8, "contiguous"), (6, 1, "single")])
def test_prefix_then_rest_equals_the_oracle(N, G, kind):
    rng = np.random.default_rng(31 + N + G)
    L = N * 16 * 2 + 7
    if kind == "contiguous":
        m = [min(G - 1, e * G // N) for e in range(N)] if G > 1 else [0] * N
    elif kind == "single":
        m = [0] * N
    else:
        m = list(range(G)) + [int(v) for v in rng.integers(0, G, N - G)]
        rng.shuffle(m)
    xs = [(rng.standard_normal(L) * 10.0 ** rng.uniform(-4, 2)).astype(np.float32) for _ in range(N)]
    want = oracle.reduce(xs, "f32")
    r = np.float32(1.0) / np.float32(N)
    C = _chunk(L, N)
    for sched in (SCHEDS if G > 1 else [es.ES_SCHED_AUTO]):
        for g in range(G):
            rows, _ = _rows(N, G, g, m, L, sched)
            for c, first, q, lo, hi in rows.tolist():
                seq = [(c + j) % N for j in range(1, N + 1)]
                assert seq[:q] == list(range(first, first + q))
                for i in range(lo, hi, max(1, (hi - lo) // 7)):
                    part = _fold(xs, seq[:q], i)             # at the stashes of the prefix
                    s = part
                    for e in seq[q:]:                         # the end fold continues (R14)
                        s = np.float32(s + xs[e][i])
                    got = np.float32(s * r)
                    assert got.view(np.uint32) == want[i].view(np.uint32), (sched, g, c, i)
    assert C > 0
