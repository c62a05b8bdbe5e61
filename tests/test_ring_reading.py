"""CPU pin of reading R2 against a ring all-reduce simulated step by
step -- the algorithm a fixed-DoP N-worker DDP ring runs, not the
oracle's formula: N ranks, bucket cut into N chunks (R1), reduce-scatter in N-1 steps where at
step s rank r sends its running partial of chunk (r - 1 - s) mod N to rank r + 1, which adds its
own contribution (fp32, one rounding per hop), then the finished chunk is scaled by fl32(1/N)
(R5) and all-gathered.  The oracle's per-element canonical fold must equal it word for word; a
ring that started chunk c anywhere else (or a zero-initialised accumulator, R3) would not.
The real-NCCL version of this check is bench.py's ring_crosscheck (multi-GPU only)."""
import numpy as np
import pytest

import oracle


def _chunk(L, N, A=16):
    per = -(-L // N)
    return -(-per // A) * A


def ring_allreduce(xs):
    N, L = len(xs), xs[0].size
    C = _chunk(L, N)
    rng = [(min(L, c * C), min(L, (c + 1) * C)) for c in range(N)]
    part = [x.astype(np.float32).copy() for x in xs]     # each rank's working buffer
    for s in range(N - 1):
        sends = []
        for r in range(N):
            c = (r - 1 - s) % N
            lo, hi = rng[c]
            sends.append(((r + 1) % N, c, part[r][lo:hi].copy()))
        for dst, c, buf in sends:
            lo, hi = rng[c]
            part[dst][lo:hi] = (buf + xs[dst][lo:hi]).astype(np.float32)   # fp32 add, one rounding
    out = np.empty(L, np.float32)
    r_ = np.float32(1.0) / np.float32(N)
    for c in range(N):                                    # rank c finished chunk c
        lo, hi = rng[c]
        out[lo:hi] = (part[c][lo:hi] * r_).astype(np.float32)
    return out


@pytest.mark.parametrize("N", [2, 3, 4, 5, 8, 12])
@pytest.mark.parametrize("L", [1, 17, 1000, 4099])
def test_canonical_fold_is_the_ring_order(N, L):
    rng = np.random.default_rng(N * 1000 + L)
    xs = [(rng.standard_normal(L) * 10.0 ** rng.uniform(-3, 3, L)).astype(np.float32) for _ in range(N)]
    got = oracle.reduce(xs, "f32")
    want = ring_allreduce(xs)
    assert np.array_equal(got.view(np.uint32), want.view(np.uint32))


def test_ring_simulation_distinguishes_start_ranks():
    """The simulation is sensitive to the reading it pins: the N = 4 rotation witness
    [2^24, 1, -2^24, 1] gives [0.5, 0.5, 0, 0.25] per chunk only with the ring's start ranks."""
    N, L = 4, 64
    xs = [np.full(L, v, np.float32) for v in (2.0 ** 24, 1.0, -(2.0 ** 24), 1.0)]
    out = ring_allreduce(xs)
    assert out[0] == 0.5 and out[16] == 0.5 and out[32] == 0.0 and out[48] == 0.25
    assert np.array_equal(out.view(np.uint32), oracle.reduce(xs, "f32").view(np.uint32))


def ring_allreduce_started(xs, shift):
    """The same ring, but every chunk's reduce-scatter starts `shift` ranks later (rank r sends
    chunk (r - 1 - shift - s) mod N at step s): chunk c is folded from rank c+1+shift on."""
    N = len(xs)
    rot = [xs[(k + shift) % N] for k in range(N)]
    out = ring_allreduce(rot)           # ring over the relabelled ranks
    return out


@pytest.mark.parametrize("N", [2, 4, 8])
def test_bench_ring_diagnostic_names_the_start_rank(N):
    """bench.py's ring_crosscheck diagnostic (ring_start_offsets) reports, per chunk, how far the
    ring's start rank is from reading R2's c+1: 0 for the R2 ring, `shift` for a shifted one.
    With two ranks every rotation is the same single (commutative) add: offsets read 0."""
    import os
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    rng = np.random.default_rng(50 + N)
    L = N * 4096
    xs = [(rng.standard_normal(L) * 10.0 ** rng.uniform(-3, 3, L)).astype(np.float32) for _ in range(N)]
    assert bench.ring_start_offsets(xs, ring_allreduce(xs)) == [0] * N
    for shift in range(1, N):
        want = [0] * N if N == 2 else [shift] * N
        assert bench.ring_start_offsets(xs, ring_allreduce_started(xs, shift)) == want
