"""Pins of the CPU oracle (oracle/) to things other than itself.

Each test pins the oracle to something the paper, a hand derivation or the
mathematics fixes:
  * hand-derived witnesses (tests/golden/*.json) for the chunk rule R1, the
    rotation R2, the first-contribution start R3, fp32 accumulation R4;
  * exact small-integer closed forms (any summation order is exact, so the
    result is the single correctly rounded product fl32(S * fl32(1/N)));
  * brute force over all N rotations on tiny inputs: each chunk must match
    exactly rotation (c+1) mod N;
  * an fp64 reference with the proved error bound (N+1)u and the north
    star's stated tolerance (1e-6 fp32, 1e-2 bf16);
  * special values (N = 1 identity, signed zero, subnormals, NaN/inf);
  * the post-scale convention R5 at N = 12, where pre-scale and divide differ;
  * the stash cast against torch's bf16 conversion (a library routine).
A plausible mistake -- dropped term, wrong start rank, off-by-one chunk,
zero-initialised accumulator, pre-scaling, per-hop bf16 rounding, FTZ --
fails at least one of these.
"""
import json
import os

import numpy as np
import pytest
import torch

import oracle

U32 = np.float32(2.0 ** -24)


def _f(s):
    """Parse a golden number: hex float, decimal, 'inf', or '0.25*fl32(3e38)'."""
    if s.startswith("0.25*fl32("):
        return np.float32(0.25) * np.float32(float(s[len("0.25*fl32("):-1]))
    if "0x" in s:
        return np.float32(float.fromhex(s))
    return np.float32(float(s))


def _bits(a):
    return np.asarray(a).view(np.uint32 if np.asarray(a).dtype == np.float32 else np.uint16)


def _bf16_bits_torch(x32):
    return torch.from_numpy(np.asarray(x32, dtype=np.float32)).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)


# ---- R1 chunk table ------------------------------------------------------------------------

def test_chunk_table_hand_cases(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "chunk_table.json")))
    for c in g["cases"]:
        C = oracle.chunk_elems(c["L"], c["N"], c["A"])
        assert C == c["C"], c
        nonempty = [(k * C, min((k + 1) * C, c["L"])) for k in range(c["N"]) if k * C < c["L"]]
        assert nonempty[-1][1] - nonempty[-1][0] == c["last_chunk"], c
        assert nonempty[-1][1] == c["L"]


def test_chunk_rule_properties():
    for L in [1, 7, 15, 16, 17, 100, 1000, 65537, 1000003]:
        for N in [1, 2, 3, 4, 7, 8, 12, 16, 32]:
            for A in [8, 16, 64]:
                C = oracle.chunk_elems(L, N, A)
                assert C % A == 0 and C * N >= L          # A-aligned, N chunks cover L
                assert C - A < -(-L // N)                 # smallest such multiple of A >= ceil(L/N)


# ---- R2/R3 rotation witnesses (hand-derived) ------------------------------------------------

def _witness_inputs(case, L, N):
    return [np.full(L, _f(v), dtype=np.float32) for v in case["x"]][:N]


def test_rotation_witness(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "witness_n4.json")))
    N, L, A, C = g["N"], g["L"], g["A"], g["chunk_elems"]
    for case in g["cases"]:
        out = oracle.reduce(_witness_inputs(case, L, N), "f32", A=A)
        for c, want in enumerate(case["out_per_chunk"]):
            w = _f(want)
            got = out[c * C:(c + 1) * C]
            assert np.all(_bits(got) == _bits(np.full(C, w, dtype=np.float32))), (case["name"], c, got[0], w)


def test_bf16_accumulates_in_fp32(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "bf16_accumulate.json")))
    xs = [_bf16_bits_torch(np.full(g["L"], _f(v), dtype=np.float32)) for v in g["x"]]
    out = oracle.reduce(xs, "bf16", A=g["A"])
    want = _bf16_bits_torch(np.full(g["L"], _f(g["out"]), dtype=np.float32))
    assert np.all(out == want)
    assert not np.all(out == _bf16_bits_torch(np.full(g["L"], _f(g["per_hop_bf16_would_give"]))))


# ---- exact small integers: closed form -------------------------------------------------------

@pytest.mark.parametrize("N", [1, 2, 3, 4, 5, 8, 12, 16, 32])
def test_small_integer_closed_form_f32(N):
    rng = np.random.default_rng(1000 + N)
    k = 24 - int(np.ceil(np.log2(N))) - 1                 # N * 2^k < 2^24: every order is exact
    L = 1000
    xs = [rng.integers(-(2 ** k), 2 ** k + 1, size=L).astype(np.float32) for _ in range(N)]
    S = np.sum(np.stack([x.astype(np.int64) for x in xs]), axis=0)      # exact integer sums
    r = np.float32(1.0) / np.float32(N)                   # IEEE-correct fl32(1/N)
    want = S.astype(np.float32) * r                       # single correctly rounded product
    out = oracle.reduce(xs, "f32")
    assert np.all(_bits(out) == _bits(want))


@pytest.mark.parametrize("N", [2, 4, 12, 32])
def test_small_integer_closed_form_bf16(N):
    rng = np.random.default_rng(2000 + N)
    L = 777
    ints = [rng.integers(-256, 257, size=L) for _ in range(N)]        # exact in bf16 (8-bit significand)
    xs = [_bf16_bits_torch(i.astype(np.float32)) for i in ints]
    S = np.sum(np.stack(ints), axis=0)
    want = _bf16_bits_torch(S.astype(np.float32) * (np.float32(1) / np.float32(N)))
    assert np.all(oracle.reduce(xs, "bf16") == want)


# ---- brute force over all rotations ---------------------------------------------------------

def _fold_from(xs, start, idx):
    N = len(xs)
    s = np.float32(xs[start][idx])
    for j in range(1, N):
        s = np.float32(s + xs[(start + j) % N][idx])
    return s


@pytest.mark.parametrize("N,L,A", [(2, 33, 8), (3, 50, 8), (4, 64, 16), (5, 61, 8), (6, 64, 8), (6, 40, 16)])
def test_bruteforce_rotation_is_c_plus_1(N, L, A):
    rng = np.random.default_rng(N * 100 + L)
    xs = [(rng.standard_normal(L) * 10.0 ** rng.uniform(-5, 2)).astype(np.float32) for _ in range(N)]
    out = oracle.reduce(xs, "f32", A=A)
    C = oracle.chunk_elems(L, N, A)
    r = np.float32(1) / np.float32(N)
    informative = 0
    for i in range(L):
        c = i // C
        cands = [np.float32(_fold_from(xs, s, i) * r) for s in range(N)]
        assert _bits(out[i]) == _bits(cands[(c + 1) % N]), (i, c)
        informative += len({int(_bits(v)) for v in cands}) > 1
    if N >= 3:                      # (N = 2: IEEE addition is commutative)
        assert informative > 0      # the data do distinguish rotations


def test_window_equals_slice():
    rng = np.random.default_rng(7)
    N, L = 5, 1003
    xs = [rng.standard_normal(L).astype(np.float32) for _ in range(N)]
    full = oracle.reduce(xs, "f32", A=16)
    for first, cnt in [(0, 10), (190, 17), (200, 401), (1000, 3)]:
        w = oracle.reduce([x[first:first + cnt] for x in xs], "f32", L=L, A=16, first=first)
        assert np.all(_bits(w) == _bits(full[first:first + cnt]))


# ---- fp64 reference and error bound ----------------------------------------------------------

@pytest.mark.parametrize("N", [4, 8, 12, 16, 32])
def test_fp64_reference_f32(N):
    rng = np.random.default_rng(3000 + N)
    L = 20000
    sig = 10.0 ** rng.uniform(-5, -2)
    mu = rng.standard_normal(L) * sig
    xs = [(mu + rng.standard_normal(L) * sig).astype(np.float32) for _ in range(N)]
    out = oracle.reduce(xs, "f32").astype(np.float64)
    X = np.stack([x.astype(np.float64) for x in xs])
    ref = X.sum(0) / N
    denom = np.abs(X).sum(0) / N
    err = np.abs(out - ref) / np.where(denom == 0, 1, denom)
    assert err.max() <= (N + 1) * float(U32) * 1.0001          # proved: fold (N-1)u + r u + product u
    assert err.max() <= 1e-6                                   # north star tolerance (fp32)
    # all-positive data, the worst case for cancellation-free accumulation
    xs = [np.abs(x) for x in xs]
    out = oracle.reduce(xs, "f32").astype(np.float64)
    X = np.abs(X)
    err = np.abs(out - X.sum(0) / N) / (X.sum(0) / N)
    assert err.max() <= (N + 1) * float(U32) * 1.0001


def test_fp64_reference_bf16_n12():
    rng = np.random.default_rng(12)
    N, L = 12, 20000
    mu = rng.standard_normal(L) * 1e-3
    x32 = [(mu + rng.standard_normal(L) * 1e-3).astype(np.float32) for _ in range(N)]
    xs = [_bf16_bits_torch(x) for x in x32]
    out = oracle.bf16_bits_to_f32(oracle.reduce(xs, "bf16")).astype(np.float64)
    X = np.stack([oracle.bf16_bits_to_f32(x).astype(np.float64) for x in xs])
    ref = X.sum(0) / N
    err = np.abs(out - ref) / (np.abs(X).sum(0) / N)
    assert err.max() <= 1e-2                                   # north star tolerance (bf16)
    assert err.max() <= 2.0 ** -8 + (N + 1) * float(U32) * 2   # one bf16 rounding + fp32 fold


def test_zero_mass_gives_exact_zero():
    N, L = 8, 64
    xs = [np.zeros(L, np.float32) for _ in range(N)]
    assert np.all(oracle.reduce(xs, "f32") == 0)


# ---- special values ----------------------------------------------------------------------------

def test_n1_is_identity_bits():
    x = np.array([0.0, -0.0, 1.5, -3.25, np.inf, -np.inf, 1e-45, -1e-45, 3.4e38, np.nan], dtype=np.float32)
    out = oracle.reduce([x], "f32")
    fin = ~np.isnan(x)
    assert np.all(_bits(out[fin]) == _bits(x[fin]))
    assert np.isnan(out[~fin]).all()
    xb = oracle.f32_to_bf16_bits(x)
    outb = oracle.reduce([xb], "bf16")
    assert np.all(outb[fin] == xb[fin])


def test_empty_bucket():
    assert oracle.reduce([np.zeros(0, np.float32)] * 3, "f32").size == 0


def test_signed_zero_and_first_contribution_start():
    N, L = 4, 16
    neg = [np.full(L, -0.0, np.float32) for _ in range(N)]
    out = oracle.reduce(neg, "f32")
    assert np.all(_bits(out) == _bits(np.full(L, -0.0, np.float32)))   # R3: a 0-initialised fold gives +0
    mixed = neg[:3] + [np.zeros(L, np.float32)]
    assert np.all(_bits(oracle.reduce(mixed, "f32")) == 0)             # (-0) + (+0) = +0


def test_subnormals_preserved():
    t = np.float32(2.0 ** -149)
    xs = [np.full(16, 2 * t, np.float32), np.full(16, 4 * t, np.float32)]
    out = oracle.reduce(xs, "f32")                                     # (2t + 4t) * 0.5 = 3t exactly
    assert np.all(out == np.float32(3) * t) and np.all(out != 0)       # FTZ/DAZ would give 0


def test_nan_inf_propagation():
    L = 16
    xs = [np.full(L, 1.0, np.float32), np.full(L, np.nan, np.float32), np.full(L, 2.0, np.float32)]
    assert np.isnan(oracle.reduce(xs, "f32")).all()
    xs = [np.full(L, np.inf, np.float32), np.full(L, -np.inf, np.float32)]
    assert np.isnan(oracle.reduce(xs, "f32")).all()
    xs = [np.full(L, np.inf, np.float32), np.full(L, 1.0, np.float32)]
    assert np.isposinf(oracle.reduce(xs, "f32")).all()


# ---- R5: post-scale by fl32(1/N), not pre-scale, not division ----------------------------------

def test_post_scale_convention_n12():
    N, L = 12, 4096
    rng = np.random.default_rng(5)
    ints = [rng.integers(-1000, 1001, size=L) for _ in range(N)]
    xs = [i.astype(np.float32) for i in ints]
    S = np.sum(np.stack(ints), axis=0)
    r = np.float32(1) / np.float32(N)
    post = S.astype(np.float32) * r                               # exact S, one rounding
    out = oracle.reduce(xs, "f32")
    assert np.all(_bits(out) == _bits(post))
    div = (S.astype(np.float64) / N).astype(np.float32)           # correctly rounded S/N
    assert np.any(_bits(div) != _bits(post))                      # the pin separates mul from div
    C = oracle.chunk_elems(L, N)
    pre = np.empty(L, np.float32)
    for i in range(L):                                            # pre-scaled fold in canonical order
        c = i // C
        s = np.float32(xs[(c + 1) % N][i] * r)
        for j in range(2, N + 1):
            s = np.float32(s + np.float32(xs[(c + j) % N][i] * r))
        pre[i] = s
    assert np.any(_bits(pre) != _bits(out))                       # ... and from pre-scaling


def test_power_of_two_equal_contributions():
    for N in [1, 2, 4, 8, 16, 32]:
        v = np.float32(1.0 + 2.0 ** -10) * np.float32(3.0)
        xs = [np.full(64, v, np.float32) for _ in range(N)]
        assert np.all(oracle.reduce(xs, "f32") == v)


def test_homogeneity_by_two():
    rng = np.random.default_rng(11)
    xs = [rng.standard_normal(500).astype(np.float32) for _ in range(7)]
    a = oracle.reduce(xs, "f32")
    b = oracle.reduce([x * np.float32(2) for x in xs], "f32")
    assert np.all(_bits(b) == _bits(a * np.float32(2)))


# ---- stash (cast) against torch ----------------------------------------------------------------

def test_stash_f32_to_bf16_matches_torch_rne():
    rng = np.random.default_rng(3)
    edge = np.array([0.0, -0.0, 1.0, 1.0 + 2 ** -8, 1.0 + 3 * 2 ** -8, 1.0 + 2 ** -8 + 2 ** -20,
                     -1.0 - 2 ** -8, 3.3895314e38, 3.4e38, -3.4e38, np.inf, -np.inf, 1e-40, -1e-40,
                     2 ** -133, 1.17549435e-38], dtype=np.float32)
    x = np.concatenate([edge, rng.standard_normal(100000).astype(np.float32) * 10.0 ** rng.uniform(-30, 30, 100000).astype(np.float32)])
    got = oracle.f32_to_bf16_bits(x)
    want = _bf16_bits_torch(x)
    assert np.all(got == want)
    nan = oracle.f32_to_bf16_bits(np.array([np.nan], np.float32))
    assert np.isnan(oracle.bf16_bits_to_f32(nan)).all()


def test_stash_bf16_to_f32_is_exact_and_identity():
    allb = np.arange(65536, dtype=np.uint32).astype(np.uint16)
    f = oracle.bf16_bits_to_f32(allb)
    want = torch.from_numpy(allb.view(np.int16)).view(torch.bfloat16).float().numpy()
    fin = ~np.isnan(want)
    assert np.all(_bits(f[fin]) == _bits(want[fin]))
    x = np.random.default_rng(0).standard_normal(1000).astype(np.float32)
    assert np.all(_bits(oracle.stash(x, "f32", "f32")) == _bits(x))
    assert np.all(oracle.stash(allb, "bf16", "bf16") == allb)


# ---- NEXT-3 compatibility variants (oracle.reduce_ex) ------------------------------------------

def test_compat_zero_is_canonical():
    rng = np.random.default_rng(50)
    for N in (3, 8, 12):
        xs = [rng.standard_normal(777).astype(np.float32) for _ in range(N)]
        assert np.all(_bits(oracle.reduce_ex(xs, "f32", 0)) == _bits(oracle.reduce(xs, "f32")))
        xb = [oracle.f32_to_bf16_bits(x) for x in xs]
        assert np.all(oracle.reduce_ex(xb, "bf16", 0) == oracle.reduce(xb, "bf16"))


def test_compat_prescale_power_of_two_identity():
    """For N = 2^k, dividing or multiplying by 1/N is exact (normal range), so
    pre-divide == pre-multiply == post-scale bit for bit."""
    rng = np.random.default_rng(51)
    for N in (2, 4, 8, 16, 32):
        xs = [(rng.standard_normal(1000) * 1e-3).astype(np.float32) for _ in range(N)]
        want = _bits(oracle.reduce(xs, "f32"))
        assert np.all(_bits(oracle.reduce_ex(xs, "f32", oracle.COMPAT_PREDIV)) == want)
        assert np.all(_bits(oracle.reduce_ex(xs, "f32", oracle.COMPAT_PREMUL)) == want)


def test_compat_prescale_closed_forms_n12():
    N, L = 12, 512
    rng = np.random.default_rng(52)
    r = np.float32(1) / np.float32(N)
    # multiples of 12: x/12 is an exact integer, every sum exact -> S/12
    ints = [rng.integers(-1000, 1001, L) * 12 for _ in range(N)]
    xs = [i.astype(np.float32) for i in ints]
    S = np.sum(np.stack(ints), 0) // 12
    assert np.all(_bits(oracle.reduce_ex(xs, "f32", oracle.COMPAT_PREDIV)) == _bits(S.astype(np.float32)))
    # one non-zero contribution per element: the fold adds +0s only
    v = (rng.standard_normal(L) * 3).astype(np.float32)
    xs = [np.zeros(L, np.float32) for _ in range(N)]
    xs[5] = v
    assert np.all(_bits(oracle.reduce_ex(xs, "f32", oracle.COMPAT_PREDIV)) == _bits(v / np.float32(N)))
    assert np.all(_bits(oracle.reduce_ex(xs, "f32", oracle.COMPAT_PREMUL)) == _bits(v * r))
    assert np.any(_bits(v / np.float32(N)) != _bits(v * r))          # the two conventions do differ


def test_compat_bf16_hop_witness(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "bf16_hop.json")))
    C = g["L"] // g["N"]
    xs = [_bf16_bits_torch(np.full(g["L"], _f(v), dtype=np.float32)) for v in g["x"]]
    hop = oracle.bf16_bits_to_f32(oracle.reduce_ex(xs, "bf16", oracle.COMPAT_BF16HOP, A=g["A"]))
    acc = oracle.bf16_bits_to_f32(oracle.reduce(xs, "bf16", A=g["A"]))
    for c in range(g["N"]):
        assert np.all(hop[c * C:(c + 1) * C] == np.float32(float(g["out_per_chunk"][c]))), c
        assert np.all(acc[c * C:(c + 1) * C] == np.float32(float(g["canonical_fp32_accumulate_per_chunk"][c]))), c


def test_compat_bf16_hop_exact_when_partials_representable():
    """Small integers whose every partial sum fits bf16's 8-bit significand:
    per-hop rounding changes nothing."""
    rng = np.random.default_rng(53)
    N = 8
    ints = [rng.integers(-15, 16, 333) for _ in range(N)]       # |partial| <= 120 < 256
    xs = [_bf16_bits_torch(i.astype(np.float32)) for i in ints]
    assert np.all(oracle.reduce_ex(xs, "bf16", oracle.COMPAT_BF16HOP) == oracle.reduce(xs, "bf16"))
    assert np.all(oracle.reduce_ex(xs, "bf16", oracle.COMPAT_BF16HOP | oracle.COMPAT_PREMUL)
                  == oracle.reduce(xs, "bf16"))                   # N = 8: 1/8 scaling exact too


# ---- NEXT-4 per-EST Philox dropout ---------------------------------------------------------------

def test_philox_known_answer_vectors(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "philox_kat.json")))
    for c in g["cases"]:
        out = oracle.philox4x32_10([int(v, 16) for v in c["ctr"]], [int(v, 16) for v in c["key"]])
        assert out == [int(v, 16) for v in c["out"]]


def test_dropout_definition_and_statistics():
    x = np.linspace(-3, 3, 40001).astype(np.float32)
    for p in (0.1, 0.5, 0.9):
        y, m = oracle.dropout(x, "f32", p, seed=123, offset=7)
        n = x.size
        keep = m.mean()
        assert abs(keep - (1 - p)) < 5 * np.sqrt(p * (1 - p) / n)          # binomial 5-sigma
        scale = np.float32(1) / (np.float32(1) - np.float32(p))
        assert np.all(_bits(y[m == 1]) == _bits(x[m == 1] * scale))
        assert np.all(_bits(y[m == 0]) == 0)                              # dropped -> +0
    # element i's decision depends only on (seed, offset, i): prefixes agree
    _, m1 = oracle.dropout(x[:1001], "f32", 0.5, 5, 9)
    _, m2 = oracle.dropout(x, "f32", 0.5, 5, 9)
    assert np.array_equal(m1, m2[:1001])
    # word i % 4 of counter i // 4: element 0..3 take the 4 output words of counter (0,0,off lo,off hi)
    w = oracle.philox4x32_10([0, 0, 9, 0], [5, 0])
    u = np.array([(v >> 8) / 16777216.0 for v in w], np.float32)
    assert np.array_equal(m2[:4], (u >= np.float32(0.5)).astype(np.uint8))
    # a new offset gives a different mask; p = 0 keeps everything
    _, m3 = oracle.dropout(x, "f32", 0.5, 5, 10)
    assert not np.array_equal(m2, m3)
    y0, m0 = oracle.dropout(x, "f32", 0.0, 5, 9)
    assert m0.all() and np.all(_bits(y0) == _bits(x))
