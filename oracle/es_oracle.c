/*
 * es_oracle.c -- plain, slow, obviously-correct CPU oracle for EasyScale's
 * placement-invariant gradient aggregation.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (libes + its Python binding) never calls it, shares no
 * code, header, table or helper with it, and fails loudly without CUDA.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:n" = line n):
 *
 *   An EasyScale job has N logical EasyScaleThreads (ESTs), each a DDP
 *   worker with a constant virtual communication rank.
 *   A global step ends when the gradients of all N ESTs are aggregated
 *   (P:526-532).  D1 "elastic determinism" demands that the aggregate is
 *   bitwise identical whatever the number of GPUs, i.e. it must
 *   equal the result of a fixed-DoP N-worker DDP all-reduce.
 *   The paper never spells out the reduction order; DESIGN.md readings
 *   R1-R6 / R13 fix it:
 *
 *     R1  chunk size  C = A * ceil(ceil(L / N) / A), chunk c = [cC, (c+1)C)
 *     R2  chunk c is folded over ranks (c+1), (c+2), ..., (c+N) mod N
 *     R3  the accumulator starts from the first contribution (not 0)
 *     R4  contributions are widened exactly to fp32; fold in fp32
 *     R5  r = fl32(1/N); result = fl32(s * r)     (post-scale)
 *     R13 then rounded once to the bucket dtype (identity for fp32,
 *         round-to-nearest-even for bf16)
 *     R6  IEEE round-to-nearest-even, subnormals kept, no FMA contraction
 *         (compiled with -O2 -ffp-contract=off, never -ffast-math)
 *
 *   There is no G and no EST->GPU mapping anywhere in this definition; that
 *   is the invariance property the GPU path must honour.
 *
 *   Stash: slot = cast(grad): identity, exact widening
 *   bf16->fp32, or RNE narrowing fp32->bf16.
 *
 * Pins: tests/test_oracle_pins.py checks this file against hand-derived
 * witnesses (tests/golden/), integer closed forms, brute force over all
 * rotations, an fp64 reference bound, and special values.
 */
#include <stdint.h>
#include <string.h>
#include <math.h>

#define ORACLE_F32 0
#define ORACLE_BF16 1

/* ------------------------------------------------------------------ */
/* scalar conversions (R4, R13)                                        */
/* ------------------------------------------------------------------ */

static float f32_from_bits(uint32_t u) { float f; memcpy(&f, &u, 4); return f; }
static uint32_t bits_from_f32(float f) { uint32_t u; memcpy(&u, &f, 4); return u; }

/* bf16 is the top 16 bits of an fp32: widening is exact. */
float es_oracle_bf16_to_f32(uint16_t h) { return f32_from_bits(((uint32_t)h) << 16); }

/* fp32 -> bf16, round to nearest, ties to even.  Written as the textbook
 * rule on the dropped 16 bits rather than the usual add-0x7FFF trick.  NaN
 * stays NaN (quiet bit set); NaNs are compared as a class (reading R7). */
uint16_t es_oracle_f32_to_bf16(float f)
{
    uint32_t u = bits_from_f32(f);
    if (isnan(f)) return (uint16_t)((u >> 16) | 0x0040u);
    uint32_t hi = u >> 16;          /* truncated result            */
    uint32_t lo = u & 0xFFFFu;      /* dropped bits                */
    if (lo > 0x8000u || (lo == 0x8000u && (hi & 1u))) hi += 1u;  /* carries into exponent -> inf ok */
    return (uint16_t)hi;
}

static float load_widened(const void *base, int32_t dtype, int64_t i)
{
    if (dtype == ORACLE_F32) return ((const float *)base)[i];
    return es_oracle_bf16_to_f32(((const uint16_t *)base)[i]);
}

static void store_rounded(void *base, int32_t dtype, int64_t i, float v)
{
    if (dtype == ORACLE_F32) ((float *)base)[i] = v;
    else ((uint16_t *)base)[i] = es_oracle_f32_to_bf16(v);
}

/* ------------------------------------------------------------------ */
/* R1: the canonical chunk size                                         */
/* ------------------------------------------------------------------ */

int64_t es_oracle_chunk_elems(int64_t L, int32_t N, int32_t A)
{
    if (L <= 0 || N <= 0 || A <= 0) return 0;
    int64_t per_rank = (L + N - 1) / N;          /* ceil(L/N)          */
    int64_t units = (per_rank + A - 1) / A;      /* ceil(ceil(L/N)/A)  */
    return units * (int64_t)A;
}

/* ------------------------------------------------------------------ */
/* a5: canonical fold + post-scale, element by element                  */
/* ------------------------------------------------------------------ */

/*
 * x[k]  : EST k's contribution to the bucket, already at element `first`
 *         (so element i of the bucket is x[k][i - first]), dtype `dtype`.
 * out   : receives elements [first, first+count) of the averaged bucket.
 * L     : the bucket's total element count (fixes the chunk table).
 * Returns 0, or -1 on bad arguments.
 */
int es_oracle_reduce(int32_t N, int64_t L, int32_t A, int32_t dtype,
                     const void *const *x, int64_t first, int64_t count, void *out)
{
    if (N <= 0 || A <= 0 || L < 0 || first < 0 || count < 0 || first + count > L) return -1;
    if (dtype != ORACLE_F32 && dtype != ORACLE_BF16) return -1;
    if (count == 0) return 0;
    const int64_t C = es_oracle_chunk_elems(L, N, A);
    const float r = 1.0f / (float)N;                      /* R5: fl32(1/N) */
    for (int64_t i = first; i < first + count; ++i) {
        const int64_t c = i / C;                          /* R1 */
        int32_t k = (int32_t)((c + 1) % N);               /* R2: start at rank c+1 */
        float s = load_widened(x[k], dtype, i - first);   /* R3: first contribution */
        for (int32_t j = 2; j <= N; ++j) {
            k = (int32_t)((c + j) % N);
            s = s + load_widened(x[k], dtype, i - first);  /* one fp32 add (R6) */
        }
        const float scaled = s * r;                       /* R5: one fp32 multiply */
        store_rounded(out, dtype, i - first, scaled);     /* R13 */
    }
    return 0;
}

/* ------------------------------------------------------------------ */
/* a1: stash (copy / cast into the EST's slot)                          */
/* ------------------------------------------------------------------ */

int es_oracle_stash(const void *src, int32_t src_dtype, void *dst, int32_t dst_dtype, int64_t n)
{
    if (n < 0) return -1;
    if ((src_dtype != ORACLE_F32 && src_dtype != ORACLE_BF16) ||
        (dst_dtype != ORACLE_F32 && dst_dtype != ORACLE_BF16)) return -1;
    for (int64_t i = 0; i < n; ++i) {
        if (src_dtype == dst_dtype) {
            if (src_dtype == ORACLE_F32) ((uint32_t *)dst)[i] = ((const uint32_t *)src)[i];
            else ((uint16_t *)dst)[i] = ((const uint16_t *)src)[i];
        } else {
            store_rounded(dst, dst_dtype, i, load_widened(src, src_dtype, i));
        }
    }
    return 0;
}

/* ------------------------------------------------------------------ */
/* NEXT-3 compatibility variants   */
/* ------------------------------------------------------------------ */

#define ORACLE_COMPAT_PREDIV 1u   /* each contribution divided by N first (DDP 1.8 div_ before all-reduce) */
#define ORACLE_COMPAT_PREMUL 2u   /* each contribution multiplied by fl32(1/N) first (NCCL ncclAvg PreMulSum) */
#define ORACLE_COMPAT_BF16HOP 4u  /* bf16 buckets: every stored intermediate rounded to bf16 (NCCL bf16 ring) */

static float round_bf16(float v) { return es_oracle_bf16_to_f32(es_oracle_f32_to_bf16(v)); }

/*
 * Same canonical order (R1-R3) as es_oracle_reduce; only the arithmetic of
 * each step changes with `compat`:
 *   v_k = widen(x[k][i]); if PREDIV: v_k = fl32(v_k / N); if PREMUL:
 *   v_k = fl32(v_k * r); if BF16HOP (bf16 only): v_k = bf16(v_k);
 *   s = v_first; s = fl32(s + v_k) [then bf16(s) if BF16HOP]; finally, if no
 *   pre-scale, s = fl32(s * r); out = round_to_dtype(s).
 * compat == 0 gives exactly es_oracle_reduce.
 */
int es_oracle_reduce_ex(int32_t N, int64_t L, int32_t A, int32_t dtype, uint32_t compat,
                        const void *const *x, int64_t first, int64_t count, void *out)
{
    if (N <= 0 || A <= 0 || L < 0 || first < 0 || count < 0 || first + count > L) return -1;
    if (dtype != ORACLE_F32 && dtype != ORACLE_BF16) return -1;
    if (compat & ~7u) return -1;
    if ((compat & ORACLE_COMPAT_PREDIV) && (compat & ORACLE_COMPAT_PREMUL)) return -1;
    if (count == 0) return 0;
    const int hop = (compat & ORACLE_COMPAT_BF16HOP) && dtype == ORACLE_BF16;
    const int pre = (compat & (ORACLE_COMPAT_PREDIV | ORACLE_COMPAT_PREMUL)) != 0;
    const int64_t C = es_oracle_chunk_elems(L, N, A);
    const float r = 1.0f / (float)N;
    for (int64_t i = first; i < first + count; ++i) {
        const int64_t c = i / C;
        float s = 0.0f;
        for (int32_t j = 1; j <= N; ++j) {
            const int32_t k = (int32_t)((c + j) % N);
            float v = load_widened(x[k], dtype, i - first);
            if (compat & ORACLE_COMPAT_PREDIV) v = v / (float)N;
            if (compat & ORACLE_COMPAT_PREMUL) v = v * r;
            if (hop) v = round_bf16(v);
            if (j == 1) s = v;
            else s = s + v;
            if (hop) s = round_bf16(s);
        }
        if (!pre) s = s * r;
        store_rounded(out, dtype, i - first, s);
    }
    return 0;
}

/* ------------------------------------------------------------------ */
/* NEXT-4: per-EST Philox dropout         */
/* ------------------------------------------------------------------ */

/* Philox4x32-10 (Salmon et al., SC'11 "Parallel random numbers: as easy as
 * 1, 2, 3"), written from its published definition: 10 rounds of
 *   (c0,c1,c2,c3) -> (hi(M1*c2) ^ c1 ^ k0, lo(M1*c2), hi(M0*c0) ^ c3 ^ k1, lo(M0*c0))
 * with the key bumped by the Weyl constants between rounds. */
void es_oracle_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4])
{
    const uint32_t M0 = 0xD2511F53u, M1 = 0xCD9E8D57u, W0 = 0x9E3779B9u, W1 = 0xBB67AE85u;
    uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
    uint32_t k0 = key[0], k1 = key[1];
    for (int round = 0; round < 10; ++round) {
        if (round > 0) { k0 += W0; k1 += W1; }
        const uint64_t p0 = (uint64_t)M0 * c0;
        const uint64_t p1 = (uint64_t)M1 * c2;
        const uint32_t n0 = (uint32_t)(p1 >> 32) ^ c1 ^ k0;
        const uint32_t n1 = (uint32_t)p1;
        const uint32_t n2 = (uint32_t)(p0 >> 32) ^ c3 ^ k1;
        const uint32_t n3 = (uint32_t)p0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/*
 * The dropout an EST's RNG context drives ("the Dropout operator
 * depends on the random number generator (RNG) states"):
 *   element i uses Philox4x32-10 with key = (seed lo, seed hi) and counter
 *   = (i/4 lo, i/4 hi, offset lo, offset hi); word w = out[i % 4];
 *   u = (w >> 8) * 2^-24;  keep = (u >= p);  scale = fl32(1 / fl32(1 - p));
 *   y = keep ? round_dtype(fl32(x * scale)) : +0;  mask[i] = keep.
 * One call consumes one offset unit (the caller advances offset by 1).
 */
int es_oracle_dropout(const void *x, void *y, uint8_t *mask, int64_t n, int32_t dtype, float p,
                      uint64_t seed, uint64_t offset)
{
    if (n < 0 || (dtype != ORACLE_F32 && dtype != ORACLE_BF16) || !(p >= 0.0f && p < 1.0f)) return -1;
    const float scale = 1.0f / (1.0f - p);
    const uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    for (int64_t i = 0; i < n; ++i) {
        const uint64_t q = (uint64_t)i >> 2;
        const uint32_t ctr[4] = {(uint32_t)q, (uint32_t)(q >> 32), (uint32_t)offset, (uint32_t)(offset >> 32)};
        uint32_t w[4];
        es_oracle_philox4x32_10(ctr, key, w);
        const float u = (float)(w[i & 3] >> 8) * (1.0f / 16777216.0f);
        const int keep = u >= p;
        if (mask) mask[i] = (uint8_t)keep;
        if (keep) store_rounded(y, dtype, i, load_widened(x, dtype, i) * scale);
        else store_rounded(y, dtype, i, 0.0f);
    }
    return 0;
}
