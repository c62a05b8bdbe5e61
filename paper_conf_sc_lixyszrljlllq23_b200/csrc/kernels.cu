// kernels.cu -- the sm_100a kernels of libes.
//
//   k_fold  : canonical-order fold + fused 1/N post-scale
//   k_stash : vectorised copy / cast into an EST's slot       (8(a) a1)
//   k_swap  : context-switch save/load of per-EST state       (8(a) a2)
//
// All three are HBM-streaming kernels (no data reuse, no contraction), so
// they use 128-bit vector loads on the non-coherent path with L1
// no-allocate (256-bit for small fp32 folds, k_fold<F32WT>), many independent
// loads in flight per thread, coalesced lanes, and grids sized in multiples
// of the 148 SMs.  Element types: F32T (4 fp32 per
// thread and source), BF16T (8 bf16; k_fold_b), F32WT (8 fp32, folds of at
// most 2^21 elements with 32-byte aligned operands).
//
// Fold and stash are MULTI-SEGMENT kernels: one launch covers many buckets
// (or many chain segments), each segment owning a contiguous range of
// blocks proportional to its size.  Fewer, larger launches remove the
// per-launch ramp-up/tail that dominated bucket-sized launches on B200.
// Launches use programmatic dependent launch (PDL): every kernel first
// waits for its predecessor (griddepcontrol.wait) and then lets its
// successor's CTAs become resident (griddepcontrol.launch_dependents), so
// the launch latency of kernel i+1 hides under the tail of kernel i while
// stream order (and therefore every data dependency) is preserved.
//
// Bit-exactness rules (R6): every fp32 add is __fadd_rn and the
// scale is __fmul_rn (no FMA contraction), no fast-math, no FTZ (nvcc
// default -ftz=false keeps subnormals), bf16 rounding is __float2bfloat16_rn
// (round to nearest even).  The value written for element i depends only on
// i and the inputs -- never on the grid, the block or which thread ran it --
// so results are launch-configuration invariant (D2 analogue).
#include "kernels.h"

#include <cuda_bf16.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <type_traits>
#include <vector>

namespace es {
namespace {

constexpr int kSMs = 148;        // B200
// Grid cap: measured on B200 (scripts/sweep_launch.py, profiles/), near
// one-shot grids (each thread ~1 vector per segment) stream better than
// persistent grid-stride ones; 148 x 64 blocks covers every bucket this build
// plans for, larger ones loop.
constexpr int kMaxBlocks = kSMs * 64;

// Device spin-waits (peer barrier, pipelined chain) trap after this long
// instead of hanging the GPU; ES_BARRIER_TIMEOUT_S overrides the 60 s default.
uint64_t barrier_timeout_ns() {
  static const uint64_t ns = [] {
    const char *e = std::getenv("ES_BARRIER_TIMEOUT_S");
    const double sec = e ? std::atof(e) : 60.0;
    return (uint64_t)((sec > 0 ? sec : 60.0) * 1e9);
  }();
  return ns;
}

bool g_pdl = [] {
  const char *e = std::getenv("ES_NO_PDL");
  return !(e && e[0] == '1');
}();

__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// ES_STASH_EARLY=0 disables the early start of stash kernels (see
// launch_stash_multi); it is on by default where the host proves it safe.
bool g_stash_early_ok = [] {
  const char *e = std::getenv("ES_STASH_EARLY");
  return !(e && e[0] == '0');
}();

__device__ __forceinline__ void pdl_enter() {
  asm volatile("griddepcontrol.wait;" ::: "memory");             // predecessor complete + visible
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");  // successor may become resident
}

__device__ __forceinline__ int4 ld_stream(const void *p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ uint2 ld_stream(const uint2 *p) {
  uint2 r;
  asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
  return r;
}
__device__ __forceinline__ int4 ld_stream(const int4 *p) { return ld_stream(static_cast<const void *>(p)); }

// L2-coherent loads (bypass L1) of data another GPU publishes during this
// kernel behind a flag (k_fold_pipe's incoming partials).
__device__ __forceinline__ int4 ld_cg(const void *p) {
  int4 r;
  asm volatile("ld.global.cg.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p)
               : "memory");
  return r;
}
__device__ __forceinline__ float ld_cg1(const float *p) {
  float r;
  asm volatile("ld.global.cg.f32 %0, [%1];" : "=f"(r) : "l"(p) : "memory");
  return r;
}

// 32-byte accesses (LDG.E.256 / STG.E.256 on sm_100a), used by the small-fold type F32WT.
struct V32 {
  int4 a, b;
};
__device__ __forceinline__ V32 ld_stream(const V32 *p) {
  V32 r;
  asm volatile("ld.global.nc.L1::no_allocate.v8.s32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(r.a.x), "=r"(r.a.y), "=r"(r.a.z), "=r"(r.a.w), "=r"(r.b.x), "=r"(r.b.y), "=r"(r.b.z),
                 "=r"(r.b.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ void st_stream(V32 *p, const V32 &v) {
  asm volatile("st.global.L1::no_allocate.v8.s32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(p), "r"(v.a.x),
               "r"(v.a.y), "r"(v.a.z), "r"(v.a.w), "r"(v.b.x), "r"(v.b.y), "r"(v.b.z), "r"(v.b.w)
               : "memory");
}

__device__ __forceinline__ void st_stream(void *p, const int4 &v) {
  asm volatile("st.global.L1::no_allocate.v4.s32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y),
               "r"(v.z), "r"(v.w)
               : "memory");
}
__device__ __forceinline__ void st_stream(uint2 *p, const uint2 &v) {
  asm volatile("st.global.L1::no_allocate.v2.u32 [%0], {%1, %2};" ::"l"(p), "r"(v.x), "r"(v.y) : "memory");
}
__device__ __forceinline__ void st_stream(int4 *p, const int4 &v) { st_stream(static_cast<void *>(p), v); }

__device__ __forceinline__ uint32_t smem_addr(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// Every kernel instantiation a launch site can reach registers its host stub
// when libes is loaded, so preload_kernels() can make CUDA's lazy loader
// (CUDA_MODULE_LOADING=LAZY, the CUDA 12 default) load them all up front: a
// first-use load cannot complete while another rank's barrier kernel spins on
// the same device, which deadlocks same-device peer ranks.
std::vector<const void *> &kernel_registry() {
  static std::vector<const void *> r;
  return r;
}
template <auto F>
struct KernelReg {
  static inline const bool token = (kernel_registry().push_back(reinterpret_cast<const void *>(F)), true);
};

template <typename K, typename P>
cudaError_t launch(K kernel, dim3 grid, dim3 block, cudaStream_t s, const P &params) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = 0;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = g_pdl ? 1 : 0;
  // Only this launch's own status: cudaGetLastError() here would report (and
  // clear) an unrelated earlier non-sticky error as this kernel's failure.
  return cudaLaunchKernelEx(&cfg, kernel, params);
}

template <auto F, typename P>
cudaError_t launch_k(dim3 grid, dim3 block, cudaStream_t s, const P &params) {
  (void)KernelReg<F>::token;
  return launch(F, grid, block, s, params);
}

// Block -> segment: the last segment whose first block is <= b.
template <typename Seg>
__device__ __forceinline__ int find_seg(const Seg *seg, int nseg, int b) {
  int lo = 0, hi = nseg - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (seg[mid].block0 <= b) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// Split `total` blocks over segments proportionally to their work (>= 1 each).
void split_blocks(const std::vector<int64_t> &work, int total, std::vector<int32_t> *block0, int *nblocks) {
  int64_t sum = 0;
  for (int64_t w : work) sum += std::max<int64_t>(w, 1);
  block0->resize(work.size());
  int b = 0;
  for (size_t i = 0; i < work.size(); ++i) {
    (*block0)[i] = b;
    int64_t nb = (int64_t)((double)total * (double)std::max<int64_t>(work[i], 1) / (double)sum + 0.5);
    b += (int)std::max<int64_t>(nb, 1);
  }
  *nblocks = b;
}

// ---- element-type traits --------------------------------------------------
// A "vector" is 16 bytes of the bucket dtype: 4 fp32 or 8 bf16.

struct F32T {
  static constexpr int kVec = 4;
  static constexpr int kSize = 4;
  static constexpr int kBatch = 8;      // sources per load batch in k_fold
  static constexpr bool kMerge = false; // opening contribution loaded alone (profiles/r02_fold_variants.md)
  using Load = int4;
  __device__ static __forceinline__ void widen(const int4 &v, float *a) {
    a[0] = __int_as_float(v.x); a[1] = __int_as_float(v.y);
    a[2] = __int_as_float(v.z); a[3] = __int_as_float(v.w);
  }
  __device__ static __forceinline__ int4 narrow(const float *a) {
    return make_int4(__float_as_int(a[0]), __float_as_int(a[1]), __float_as_int(a[2]),
                     __float_as_int(a[3]));
  }
  __device__ static __forceinline__ float load1(const void *p, int64_t i) {
    return reinterpret_cast<const float *>(p)[i];
  }
  __device__ static __forceinline__ void store1(void *p, int64_t i, float v) {
    reinterpret_cast<float *>(p)[i] = v;
  }
};

struct BF16T {
  static constexpr int kVec = 8;
  static constexpr int kSize = 2;
  static constexpr int kBatch = 8;
  static constexpr bool kMerge = true;  // opening contribution in the first batch (+2.4 % BERT fold)
  using Load = int4;
  // bf16 is the high half of an fp32: widening is exact (R4).
  __device__ static __forceinline__ void widen2(uint32_t w, float *a) {
    a[0] = __uint_as_float(w << 16);
    a[1] = __uint_as_float(w & 0xFFFF0000u);
  }
  __device__ static __forceinline__ void widen(const int4 &v, float *a) {
    widen2((uint32_t)v.x, a + 0); widen2((uint32_t)v.y, a + 2);
    widen2((uint32_t)v.z, a + 4); widen2((uint32_t)v.w, a + 6);
  }
  __device__ static __forceinline__ uint32_t pack2(float lo, float hi) {   // RNE (R13)
    uint32_t l = __bfloat16_as_ushort(__float2bfloat16_rn(lo));
    uint32_t h = __bfloat16_as_ushort(__float2bfloat16_rn(hi));
    return l | (h << 16);
  }
  __device__ static __forceinline__ int4 narrow(const float *a) {
    return make_int4((int)pack2(a[0], a[1]), (int)pack2(a[2], a[3]), (int)pack2(a[4], a[5]),
                     (int)pack2(a[6], a[7]));
  }
  __device__ static __forceinline__ float load1(const void *p, int64_t i) {
    return __uint_as_float(((uint32_t) reinterpret_cast<const unsigned short *>(p)[i]) << 16);
  }
  __device__ static __forceinline__ void store1(void *p, int64_t i, float v) {
    reinterpret_cast<unsigned short *>(p)[i] = __bfloat16_as_ushort(__float2bfloat16_rn(v));
  }
};

// fp32, 8 elements (32 bytes) per thread and source: the small-fold type.  A fold of at most
// kWideMaxElems elements is latency-bound (1M fp32 = 1.7 waves of one-vector threads); F32WT
// halves the threads to one wave and, with the opening contribution in the first batch, needs
// one memory round trip per thread (launch_fold_multi picks it; same per-element arithmetic).
struct F32WT {
  static constexpr int kVec = 8;
  static constexpr int kSize = 4;
  static constexpr int kBatch = 4;      // 4 x 32 B in flight: the registers of F32T's 8 x 16 B
  static constexpr bool kMerge = true;
  using Load = V32;
  __device__ static __forceinline__ void widen(const V32 &v, float *a) {
    F32T::widen(v.a, a);
    F32T::widen(v.b, a + 4);
  }
  __device__ static __forceinline__ V32 narrow(const float *a) { return V32{F32T::narrow(a), F32T::narrow(a + 4)}; }
  __device__ static __forceinline__ float load1(const void *p, int64_t i) { return F32T::load1(p, i); }
  __device__ static __forceinline__ void store1(void *p, int64_t i, float v) { F32T::store1(p, i, v); }
};
constexpr int64_t kWideMaxElems = 1 << 21;

// ---- k_fold ---------------------------------------------------------------

struct FoldSeg {
  const float *part_in;   // element lo at part_in[0], or null
  void *out;              // element lo at out[0]
  int64_t lo, n;
  uint32_t C;
  int32_t rot, m, src0;   // sources: src[src0 ...]
  int32_t out_partial;
  int32_t block0;         // first block of this segment
  int32_t npush;          // ES_OPT_PEER_PUSH: extra copies of the final result, pointers in src[] after the sources
};

template <int MAXSEG, int MAXSRC>
struct FoldParams {
  int32_t nseg, N, nblocks;
  float r;
  uint32_t compat;        // NEXT-3 variant bits (COMPAT kernels only)
  FoldSeg seg[MAXSEG];
  const void *src[MAXSRC];
};

// NEXT-3 compatibility variants: the
// canonical order is unchanged; only each step's arithmetic differs.
constexpr uint32_t kPreDiv = 1, kPreMul = 2, kBf16Hop = 4;

__device__ __forceinline__ float round_bf16(float v) { return __bfloat162float(__float2bfloat16_rn(v)); }

// A widened contribution as the variant sees it (pre-scale, bf16 storage).
template <bool COMPAT>
__device__ __forceinline__ float prep(float v, uint32_t compat, float r, float fN) {
  if (COMPAT) {
    if (compat & kPreDiv) v = __fdiv_rn(v, fN);
    if (compat & kPreMul) v = __fmul_rn(v, r);
    if (compat & kBf16Hop) v = round_bf16(v);
  }
  return v;
}

template <bool COMPAT>
__device__ __forceinline__ float add_step(float s, float v, uint32_t compat) {
  s = __fadd_rn(s, v);
  if (COMPAT && (compat & kBf16Hop)) s = round_bf16(s);
  return s;
}

// Fold of one 16-byte vector at segment offset t (elements), into acc[V].
template <typename T, bool COMPAT, bool CG = false>
__device__ __forceinline__ void fold_vector(const FoldSeg &g, const void *const *src, int32_t N, int64_t t,
                                            float *acc, uint32_t compat, float r) {
  const float fN = (float)N;
  constexpr int V = T::kVec;
  int cnt, idx;
  if (g.rot) {
    const uint32_t c = (uint32_t)(g.lo + t) / g.C;           // R1: chunk of this vector
    idx = (int)(c + 1u == (uint32_t)N ? 0u : c + 1u);         // R2: start at rank c+1
    cnt = N;
  } else {
    idx = 0;
    cnt = g.m;
  }
  const int64_t boff = t * T::kSize;
  // R3 / R14: the accumulator opens with the first contribution, or continues a chain partial.
  // bf16 (MERGE): the opening contribution is loaded in the first batch together with the next
  // ones -- one memory round trip for up to kBatch sources instead of a dependent one first;
  // measured +2.8 % on BERT's fold (profiles/r02_fold_variants.md).  fp32 keeps the separate
  // opening load, which measured 1.9-2.1 % faster there (Swin-B, VGG-19).  Same adds, same order.
  constexpr bool MERGE = T::kMerge;
  constexpr int KB = T::kBatch;
  using LD = typename T::Load;
  bool open = g.part_in == nullptr;
  int done = 0;
  if (!open) {
    const float *pp = g.part_in + t;
#pragma unroll
    for (int q = 0; q < V / 4; ++q) {
      int4 w = CG ? ld_cg(pp + 4 * q) : ld_stream(pp + 4 * q);
      acc[4 * q + 0] = __int_as_float(w.x); acc[4 * q + 1] = __int_as_float(w.y);
      acc[4 * q + 2] = __int_as_float(w.z); acc[4 * q + 3] = __int_as_float(w.w);
    }
  } else if (!MERGE) {
    LD w = ld_stream(reinterpret_cast<const LD *>(reinterpret_cast<const char *>(src[idx]) + boff));
    T::widen(w, acc);
#pragma unroll
    for (int e = 0; e < V; ++e) acc[e] = prep<COMPAT>(acc[e], compat, r, fN);
    idx = (idx + 1 == cnt) ? 0 : idx + 1;
    done = 1;
    open = false;
  }
  while (done < cnt) {
    const int nb = min(KB, cnt - done);
    LD buf[KB];
    int k = idx;
#pragma unroll
    for (int b = 0; b < KB; ++b) {                            // all loads of the batch first ...
      if (b < nb) {
        buf[b] = ld_stream(reinterpret_cast<const LD *>(reinterpret_cast<const char *>(src[k]) + boff));
        k = (k + 1 == cnt) ? 0 : k + 1;
      }
    }
#pragma unroll
    for (int b = 0; b < KB; ++b) {                            // ... then the adds, in canonical order
      if (b < nb) {
        float x[V];
        T::widen(buf[b], x);
        if (MERGE && b == 0 && open) {                        // R3: start from the first contribution
#pragma unroll
          for (int e = 0; e < V; ++e) acc[e] = prep<COMPAT>(x[e], compat, r, fN);
        } else {
#pragma unroll
          for (int e = 0; e < V; ++e) acc[e] = add_step<COMPAT>(acc[e], prep<COMPAT>(x[e], compat, r, fN), compat);
        }
      }
    }
    open = false;
    idx = k;
    done += nb;
  }
}

template <typename T, bool COMPAT, bool CG = false>
__device__ __forceinline__ float fold_scalar(const FoldSeg &g, const void *const *src, int32_t N, int64_t t,
                                             uint32_t compat, float r) {
  const float fN = (float)N;
  int cnt, idx;
  if (g.rot) {
    const uint32_t c = (uint32_t)(g.lo + t) / g.C;
    idx = (int)(c + 1u == (uint32_t)N ? 0u : c + 1u);
    cnt = N;
  } else {
    idx = 0;
    cnt = g.m;
  }
  float s;
  int done = 0;
  if (g.part_in) {
    s = CG ? ld_cg1(g.part_in + t) : g.part_in[t];
  } else {
    s = prep<COMPAT>(T::load1(src[idx], t), compat, r, fN);
    idx = (idx + 1 == cnt) ? 0 : idx + 1;
    done = 1;
  }
  for (; done < cnt; ++done) {
    s = add_step<COMPAT>(s, prep<COMPAT>(T::load1(src[idx], t), compat, r, fN), compat);
    idx = (idx + 1 == cnt) ? 0 : idx + 1;
  }
  return s;
}

template <typename T, int MAXSEG, int MAXSRC, bool COMPAT>
__device__ __forceinline__ void fold_body(const FoldParams<MAXSEG, MAXSRC> &p) {
  constexpr int V = T::kVec;
  // post-scale unless a pre-scale variant already applied 1/N (R5 vs NEXT-3)
  const bool post = !COMPAT || !(p.compat & (kPreDiv | kPreMul));
  pdl_enter();
  const int si = find_seg(p.seg, p.nseg, (int)blockIdx.x);
  const FoldSeg &g = p.seg[si];
  const int nb = (si + 1 < p.nseg ? p.seg[si + 1].block0 : p.nblocks) - g.block0;
  const void *const *src = p.src + g.src0;
  const int cnt_src = g.rot ? p.N : g.m;                             // push pointers follow the sources
  const int64_t nvec = g.n / V;
  const int64_t tid0 = (int64_t)(blockIdx.x - g.block0) * blockDim.x + threadIdx.x;
  const int64_t stride = (int64_t)nb * blockDim.x;
  for (int64_t v = tid0; v < nvec; v += stride) {
    const int64_t t = v * V;
    float acc[V];
    fold_vector<T, COMPAT>(g, src, p.N, t, acc, p.compat, p.r);
    if (g.out_partial) {
      float *o = reinterpret_cast<float *>(g.out) + t;
#pragma unroll
      for (int q = 0; q < V / 4; ++q)
        st_stream(o + 4 * q, make_int4(__float_as_int(acc[4 * q]), __float_as_int(acc[4 * q + 1]),
                                       __float_as_int(acc[4 * q + 2]), __float_as_int(acc[4 * q + 3])));
    } else {
      if (post) {
#pragma unroll
        for (int e = 0; e < V; ++e) acc[e] = __fmul_rn(acc[e], p.r);   // R5: one rounding
      }
      using LD = typename T::Load;
      const LD w = T::narrow(acc);                                     // R13
      st_stream(reinterpret_cast<LD *>(reinterpret_cast<char *>(g.out) + t * T::kSize), w);
      // ES_OPT_PEER_PUSH: the same words into every peer's RESULT area over NVLink (posted
      // stores), so the all-gather's traffic rides the fold's otherwise idle egress
      for (int j = 0; j < g.npush; ++j)
        st_stream(reinterpret_cast<LD *>(reinterpret_cast<char *>(const_cast<void *>(src[cnt_src + j])) + t * T::kSize), w);
    }
  }
  const int64_t tail0 = nvec * V;                                    // ragged tail (< V elements)
  if (tid0 < g.n - tail0) {
    const int64_t t = tail0 + tid0;
    const float s = fold_scalar<T, COMPAT>(g, src, p.N, t, p.compat, p.r);
    if (g.out_partial) {
      reinterpret_cast<float *>(g.out)[t] = s;
    } else {
      const float o = post ? __fmul_rn(s, p.r) : s;
      T::store1(g.out, t, o);
      for (int j = 0; j < g.npush; ++j) T::store1(const_cast<void *>(src[cnt_src + j]), t, o);
    }
  }
}

// fp32: compiled as in round 1 (62 registers, no bound).  bf16 (k_fold_b): at most 64 registers
// (4 resident 256-thread blocks per SM) -- the merged first batch otherwise takes 79 and drops to
// 3 (profiles/r02_fold_variants.md).
template <typename T, int MAXSEG, int MAXSRC, bool COMPAT>
__global__ void __launch_bounds__(256) k_fold(const __grid_constant__ FoldParams<MAXSEG, MAXSRC> p) {
  fold_body<T, MAXSEG, MAXSRC, COMPAT>(p);
}
template <typename T, int MAXSEG, int MAXSRC, bool COMPAT>
__global__ void __launch_bounds__(256, 4) k_fold_b(const __grid_constant__ FoldParams<MAXSEG, MAXSRC> p) {
  fold_body<T, MAXSEG, MAXSRC, COMPAT>(p);
}

// ---- k_fold_pipe: the PEER_CHAIN rounds as one tile-pipelined kernel ----------------
// Every chain segment on this GPU (all rounds, all buckets of one dtype) is cut
// into tiles of kPipeTile elements; CTAs take tiles from an atomic ticket in
// (round, bucket, chunk, tile) order.  A tile of a segment that continues a
// partial first waits until the producer GPU has published that tile
// (system-scope acquire on the producer's flag, read over NVLink), folds its
// local contributions onto it and, if the chunk continues on another GPU,
// publishes its own tile (system-scope release).  Round r+1 of a chunk thus
// starts on tile 0 while round r is still folding later tiles: the partial's
// transfer overlaps the folds tile by tile, with no device-wide barrier between
// rounds.  Forward progress: on every GPU the tickets of round r are all taken
// before any of round r+1 and round 0 waits for nothing (induction on r).
// Flag value v = the epoch the step's closing barrier will publish, read from
// this rank's device epoch counter: identical on every rank and larger than
// any value of an earlier step.

struct PipeSeg {
  FoldSeg f;              // f.block0 unused
  const uint64_t *wait;   // producer's flags for this chunk's previous round (tile t: wait[t]), or null
  uint64_t *pub;          // own flags for this round (tile t: pub[t]), or null (the chunk ends here)
  int32_t tile0;          // first ticket of this segment
};

template <int MAXSEG, int MAXSRC>
struct PipeParams {
  int32_t nseg, N, ntiles;
  float r;
  const uint64_t *epoch;  // this rank's barrier epoch counter
  unsigned int *ticket;   // zeroed before the launch
  uint64_t timeout_ns;
  PipeSeg seg[MAXSEG];
  const void *src[MAXSRC];
};

__device__ __forceinline__ int find_tile_seg(const PipeSeg *seg, int nseg, int tk) {
  int lo = 0, hi = nseg - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (seg[mid].tile0 <= tk) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

template <typename T, int MAXSEG, int MAXSRC>
__global__ void __launch_bounds__(256) k_fold_pipe(const __grid_constant__ PipeParams<MAXSEG, MAXSRC> p) {
  constexpr int V = T::kVec;
  static_assert(kPipeTile % (4 * V) == 0, "tiles hold whole vectors");
  __shared__ int s_tk;
  // Wait for the predecessor but never let the successor (the closing
  // barrier) become resident early: a dependent grid parked on the SMs while
  // these CTAs spin on peers was measured to stall same-device peers
  // (loopback) until the timeout; the successor launches at completion.
  pdl_wait();
  const uint64_t v = *reinterpret_cast<const volatile uint64_t *>(p.epoch) + 1;
  for (;;) {
    if (threadIdx.x == 0) s_tk = (int)atomicAdd(p.ticket, 1u);
    __syncthreads();
    const int tk = s_tk;
    __syncthreads();                                   // s_tk is rewritten next iteration
    if (tk >= p.ntiles) break;
    const PipeSeg &ps = p.seg[find_tile_seg(p.seg, p.nseg, tk)];
    const FoldSeg &g = ps.f;
    const int64_t tile = tk - ps.tile0;
    const int64_t e0 = tile * kPipeTile, e1 = min(g.n, e0 + (int64_t)kPipeTile);
    if (ps.wait && threadIdx.x == 0) {                 // the producer's tile, published over NVLink
      const uint64_t *fl = ps.wait + tile;
      uint64_t f = 0, t0 = 0, now = 0;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
      for (;;) {
        asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(f) : "l"(fl) : "memory");
        if (f >= v) break;
        __nanosleep(64);
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
        if (now - t0 > p.timeout_ns) __trap();         // the producer never published: fail loudly
      }
    }
    __syncthreads();
    const void *const *src = p.src + g.src0;
    const int64_t tail0 = (g.n / V) * V;
    const int64_t vend = min(e1, tail0);
    for (int64_t t = e0 + (int64_t)threadIdx.x * V; t < vend; t += (int64_t)blockDim.x * V) {
      float acc[V];
      fold_vector<T, false, true>(g, src, p.N, t, acc, 0u, p.r);
      if (g.out_partial) {
        float *o = reinterpret_cast<float *>(g.out) + t;
#pragma unroll
        for (int q = 0; q < V / 4; ++q)
          st_stream(o + 4 * q, make_int4(__float_as_int(acc[4 * q]), __float_as_int(acc[4 * q + 1]),
                                         __float_as_int(acc[4 * q + 2]), __float_as_int(acc[4 * q + 3])));
      } else {
#pragma unroll
        for (int e = 0; e < V; ++e) acc[e] = __fmul_rn(acc[e], p.r);   // R5: one rounding
        st_stream(reinterpret_cast<char *>(g.out) + t * T::kSize, T::narrow(acc));  // R13
      }
    }
    if (e1 == g.n && tail0 < g.n && (int64_t)threadIdx.x < g.n - tail0) {   // ragged tail, last tile
      const int64_t t = tail0 + threadIdx.x;
      const float sc = fold_scalar<T, false, true>(g, src, p.N, t, 0u, p.r);
      if (g.out_partial) reinterpret_cast<float *>(g.out)[t] = sc;
      else T::store1(g.out, t, __fmul_rn(sc, p.r));
    }
    if (ps.pub) {                                      // publish this tile to the next GPU
      __syncthreads();
      if (threadIdx.x == 0) {
        __threadfence_system();
        asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(ps.pub + tile), "l"(v) : "memory");
      }
    }
  }
}

// ---- k_fold_tma: TMA / shared-memory staged fold (experiment) -------------------
// The north star's "pulls the N EST contributions through TMA/shared-memory
// staging": per tile of 256*V elements one elected thread issues N
// cp.async.bulk copies (one per source row, completion on the stage's
// mbarrier), all threads fold from shared memory in canonical order and
// store.  S-stage ring, tiles prefetched S-1 ahead.  Canonical (rot)
// segments without partials only, N <= 16.  Selected with ES_FOLD_TMA=1;
// the LDG kernel above is the default (profiles/: it measured as fast).

template <typename T, int MAXSEG, int MAXSRC, int S>
__global__ void __launch_bounds__(256) k_fold_tma(const __grid_constant__ FoldParams<MAXSEG, MAXSRC> p) {
  constexpr int V = T::kVec;
  constexpr int TILE = 256 * V;                 // elements per tile
  constexpr int TILEB = TILE * T::kSize;        // 4096 bytes per source row
  extern __shared__ __align__(128) unsigned char ring[];
  __shared__ __align__(8) uint64_t full[S];
  pdl_enter();
  const int si = find_seg(p.seg, p.nseg, (int)blockIdx.x);
  const FoldSeg &g = p.seg[si];
  const int nb = (si + 1 < p.nseg ? p.seg[si + 1].block0 : p.nblocks) - g.block0;
  const int lb = (int)blockIdx.x - g.block0;
  const void *const *src = p.src + g.src0;
  const int N = p.N;
  const int64_t ntiles = (g.n + TILE - 1) / TILE;
  const int tid = threadIdx.x;
  if (tid == 0) {
    for (int st = 0; st < S; ++st)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&full[st])) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int64_t i) {                 // thread 0: tile number i of this block
    const int64_t tile = lb + i * nb;
    const int st = (int)(i % S);
    const int64_t t0 = tile * TILE;
    const int64_t cnt = min((int64_t)TILE, g.n - t0);
    const uint32_t bytes = (uint32_t)((cnt * T::kSize) & ~int64_t(15));
    const uint32_t bar = smem_addr(&full[st]);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes * (uint32_t)N)
                 : "memory");
    if (bytes == 0) return;
    for (int k = 0; k < N; ++k)
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(smem_addr(ring + ((size_t)st * N + k) * TILEB)),
                   "l"(reinterpret_cast<const char *>(src[k]) + t0 * T::kSize), "r"(bytes), "r"(bar)
                   : "memory");
  };
  int64_t mine = lb < ntiles ? (ntiles - lb + nb - 1) / nb : 0;
  if (tid == 0)
    for (int64_t i = 0; i < S - 1 && i < mine; ++i) issue(i);
  for (int64_t i = 0; i < mine; ++i) {
    if (tid == 0 && i + S - 1 < mine) issue(i + S - 1);
    const int st = (int)(i % S);
    const uint32_t bar = smem_addr(&full[st]);
    const uint32_t parity = (uint32_t)((i / S) & 1);
    uint32_t ok = 0;
    do {
      asm volatile("{\n .reg .pred q;\n mbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2;\n selp.u32 %0, 1, 0, q;\n}"
                   : "=r"(ok)
                   : "r"(bar), "r"(parity)
                   : "memory");
    } while (!ok);
    const int64_t t0 = (lb + i * nb) * TILE;
    const int64_t cnt = min((int64_t)TILE, g.n - t0);
    const int e0 = tid * V;
    if (e0 + V <= cnt) {
      const uint32_t c = (uint32_t)(g.lo + t0 + e0) / g.C;    // R1
      int k = (int)(c + 1u == (uint32_t)N ? 0u : c + 1u);      // R2
      float acc[V];
      const unsigned char *row0 = ring + (size_t)st * N * TILEB + (size_t)e0 * T::kSize;
      T::widen(*reinterpret_cast<const int4 *>(row0 + (size_t)k * TILEB), acc);   // R3
      for (int j = 1; j < N; ++j) {
        k = (k + 1 == N) ? 0 : k + 1;
        float x[V];
        T::widen(*reinterpret_cast<const int4 *>(row0 + (size_t)k * TILEB), x);
#pragma unroll
        for (int e = 0; e < V; ++e) acc[e] = __fadd_rn(acc[e], x[e]);
      }
#pragma unroll
      for (int e = 0; e < V; ++e) acc[e] = __fmul_rn(acc[e], p.r);                  // R5
      st_stream(reinterpret_cast<char *>(g.out) + (t0 + e0) * T::kSize, T::narrow(acc));
    } else if (e0 < cnt) {                                      // ragged tail of the segment
      for (int64_t t = t0 + e0; t < t0 + cnt; ++t)
        T::store1(g.out, t, __fmul_rn(fold_scalar<T, false>(g, src, N, t, 0u, p.r), p.r));
    }
    __syncthreads();                                            // stage free for the refill
  }
}

int g_fold_tma = [] {
  const char *e = std::getenv("ES_FOLD_TMA");
  return e ? std::atoi(e) : 0;
}();

template <typename T, int MAXSEG, int MAXSRC>
cudaError_t launch_fold_group(int32_t N, float r, uint32_t compat, const FoldSegDesc *d, int nseg, cudaStream_t s,
                              int bo, int to) {
  FoldParams<MAXSEG, MAXSRC> p;
  p.nseg = nseg;
  p.N = N;
  p.r = r;
  p.compat = compat;
  int nsrc = 0;
  std::vector<int64_t> work(nseg);
  for (int i = 0; i < nseg; ++i) {
    FoldSeg &g = p.seg[i];
    const int k = d[i].rot ? N : d[i].m;
    g.part_in = d[i].part_in;
    g.out = d[i].out;
    g.lo = d[i].lo;
    g.n = d[i].n;
    g.C = d[i].C;
    g.rot = d[i].rot ? 1 : 0;
    g.m = d[i].m;
    g.src0 = nsrc;
    g.out_partial = d[i].out_partial ? 1 : 0;
    g.npush = d[i].npush;
    for (int j = 0; j < k; ++j) p.src[nsrc + j] = d[i].src[j];
    for (int j = 0; j < d[i].npush; ++j) p.src[nsrc + k + j] = d[i].push[j];
    nsrc += k + d[i].npush;
    work[i] = (d[i].n + T::kVec - 1) / T::kVec * (int64_t)(k + 1 + d[i].npush);   // vectors x streams
  }
  const int threads = to > 0 ? to : 256;
  int64_t vecs = 0;
  for (int i = 0; i < nseg; ++i) vecs += (d[i].n + T::kVec - 1) / T::kVec;
  int total = (int)std::min<int64_t>((vecs + threads - 1) / threads, (int64_t)kMaxBlocks);
  if (bo > 0) total = bo;
  else if (bo < 0) total = std::min(total, -bo);   // a cap (ES_OPT_STASH_BACKGROUND)
  total = std::max(total, nseg);
  std::vector<int32_t> block0;
  split_blocks(work, total, &block0, &p.nblocks);
  for (int i = 0; i < nseg; ++i) p.seg[i].block0 = block0[i];
  if constexpr (std::is_same<T, F32WT>::value) {   // small canonical folds only (launch_fold_multi)
    return launch_k<k_fold<T, MAXSEG, MAXSRC, false>>(dim3(p.nblocks), dim3(threads), s, p);
  } else {
  bool tma_ok = g_fold_tma > 0 && !compat && N <= 16 && bo == 0 && to == 0;
  for (int i = 0; i < nseg && tma_ok; ++i) tma_ok = d[i].rot && !d[i].part_in && !d[i].out_partial && !d[i].npush;
  if (tma_ok) {
    constexpr int kS = 3;
    const int stage = N * 256 * T::kVec * T::kSize;
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(k_fold_tma<T, MAXSEG, MAXSRC, kS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           kS * 16 * 4096);
      attr = true;
    }
    const int per_sm = std::max(1, (227 * 1024) / (kS * stage + 1024));
    int64_t tiles = 0;
    for (int i = 0; i < nseg; ++i) tiles += (d[i].n + 256 * T::kVec - 1) / (256 * T::kVec);
    const int grid = (int)std::max<int64_t>(nseg, std::min<int64_t>(tiles, (int64_t)kSMs * per_sm));
    split_blocks(work, grid, &block0, &p.nblocks);
    for (int i = 0; i < nseg; ++i) p.seg[i].block0 = block0[i];
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(p.nblocks);
    cfg.blockDim = dim3(256);
    cfg.dynamicSmemBytes = kS * stage;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = g_pdl ? 1 : 0;
    (void)KernelReg<k_fold_tma<T, MAXSEG, MAXSRC, kS>>::token;
    return cudaLaunchKernelEx(&cfg, k_fold_tma<T, MAXSEG, MAXSRC, kS>, p);
  }
  if constexpr (T::kSize == 2) {
    if (compat) return launch_k<k_fold_b<T, MAXSEG, MAXSRC, true>>(dim3(p.nblocks), dim3(threads), s, p);
    return launch_k<k_fold_b<T, MAXSEG, MAXSRC, false>>(dim3(p.nblocks), dim3(threads), s, p);
  } else {
    if (compat) return launch_k<k_fold<T, MAXSEG, MAXSRC, true>>(dim3(p.nblocks), dim3(threads), s, p);
    return launch_k<k_fold<T, MAXSEG, MAXSRC, false>>(dim3(p.nblocks), dim3(threads), s, p);
  }
  }
}

template <typename T>
cudaError_t launch_fold_t(int32_t N, float r, uint32_t compat, const FoldSegDesc *segs, int nseg, cudaStream_t s,
                          int bo, int to, int *launches) {
  constexpr int kSmallSeg = 4, kSmallSrc = 64, kBigSeg = 64, kBigSrc = 1024;
  int i = 0;
  while (i < nseg) {
    int j = i, nsrc = 0;                     // greedy group within the large capacity
    while (j < nseg) {
      const int k = (segs[j].rot ? N : segs[j].m) + segs[j].npush;
      if (j - i + 1 > kBigSeg || nsrc + k > kBigSrc) break;
      nsrc += k;
      ++j;
    }
    if (j == i) return cudaErrorInvalidValue;   // one segment with > 1024 sources (N <= 1024 by contract)
    cudaError_t e = (j - i <= kSmallSeg && nsrc <= kSmallSrc)
                        ? launch_fold_group<T, kSmallSeg, kSmallSrc>(N, r, compat, segs + i, j - i, s, bo, to)
                        : launch_fold_group<T, kBigSeg, kBigSrc>(N, r, compat, segs + i, j - i, s, bo, to);
    if (e != cudaSuccess) return e;
    ++*launches;
    i = j;
  }
  return cudaSuccess;
}


template <typename T, int MAXSEG, int MAXSRC>
cudaError_t launch_pipe_group(int32_t N, float r, const PipeSegDesc *d, int nseg, const uint64_t *epoch,
                              unsigned int *ticket, int share, cudaStream_t s) {
  PipeParams<MAXSEG, MAXSRC> p;
  p.nseg = nseg;
  p.N = N;
  p.r = r;
  p.epoch = epoch;
  p.ticket = ticket;
  p.timeout_ns = barrier_timeout_ns();
  int nsrc = 0, tiles = 0;
  for (int i = 0; i < nseg; ++i) {
    PipeSeg &g = p.seg[i];
    const FoldSegDesc &f = d[i].f;
    g.f.part_in = f.part_in;
    g.f.out = f.out;
    g.f.lo = f.lo;
    g.f.n = f.n;
    g.f.C = f.C;
    g.f.rot = 0;
    g.f.m = f.m;
    g.f.src0 = nsrc;
    g.f.out_partial = f.out_partial ? 1 : 0;
    g.f.block0 = 0;
    g.f.npush = 0;          // k_fold_pipe never pushes (ES_OPT_PEER_PUSH applies to k_fold launches)
    for (int j = 0; j < f.m; ++j) p.src[nsrc + j] = f.src[j];
    nsrc += f.m;
    g.wait = d[i].wait;
    g.pub = d[i].pub;
    g.tile0 = tiles;
    tiles += (int)((f.n + kPipeTile - 1) / kPipeTile);
  }
  p.ntiles = tiles;
  static const int occ = [] {
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_fold_pipe<T, MAXSEG, MAXSRC>, 256, 0) != cudaSuccess) {
      cudaGetLastError();
      b = 1;
    }
    return std::max(b, 1);
  }();
  const int grid = std::max(1, std::min(tiles, kSMs * occ / std::max(share, 1)));
  cudaError_t e = cudaMemsetAsync(ticket, 0, sizeof(unsigned int), s);
  if (e != cudaSuccess) return e;
  return launch_k<k_fold_pipe<T, MAXSEG, MAXSRC>>(dim3(grid), dim3(256), s, p);
}

template <typename T>
cudaError_t launch_pipe_t(int32_t N, float r, const PipeSegDesc *segs, int nseg, const uint64_t *epoch,
                          unsigned int *ticket, int share, cudaStream_t s, int *launches) {
  constexpr int kSeg = 64, kSrc = 1024;
  int i = 0;
  while (i < nseg) {                                   // groups keep the (round-major) order
    int j = i, nsrc = 0;
    while (j < nseg && j - i < kSeg && nsrc + segs[j].f.m <= kSrc) nsrc += segs[j++].f.m;
    if (j == i) return cudaErrorInvalidValue;
    cudaError_t e = launch_pipe_group<T, kSeg, kSrc>(N, r, segs + i, j - i, epoch, ticket, share, s);
    if (e != cudaSuccess) return e;
    ++*launches;
    i = j;
  }
  return cudaSuccess;
}

// ---- k_stash ----------------------------------------------------------------
// Each lane moves one "unit" of E elements per access: E = 4 when a cast is
// involved (fp32 16 B <-> bf16 8 B), else one 16-byte vector.  Consecutive
// lanes take consecutive units, so every warp-wide load and store covers
// one contiguous span (fully coalesced).  kU units per thread per
// iteration, spaced by the segment's grid stride, all loads before stores.

template <int BYTES> struct VecT;
template <> struct VecT<16> { using T = int4; };
template <> struct VecT<8> { using T = uint2; };

template <typename S, typename D, int E>
struct Cast;
template <> struct Cast<F32T, F32T, 4> {
  __device__ static __forceinline__ int4 apply(const int4 &v) { return v; }
};
template <> struct Cast<BF16T, BF16T, 8> {
  __device__ static __forceinline__ int4 apply(const int4 &v) { return v; }
};
template <> struct Cast<F32T, BF16T, 4> {             // RNE narrowing
  __device__ static __forceinline__ uint2 apply(const int4 &v) {
    return make_uint2(BF16T::pack2(__int_as_float(v.x), __int_as_float(v.y)),
                      BF16T::pack2(__int_as_float(v.z), __int_as_float(v.w)));
  }
};
template <> struct Cast<BF16T, F32T, 4> {             // exact widening
  __device__ static __forceinline__ int4 apply(const uint2 &v) {
    float a[4];
    BF16T::widen2(v.x, a);
    BF16T::widen2(v.y, a + 2);
    return make_int4(__float_as_int(a[0]), __float_as_int(a[1]), __float_as_int(a[2]), __float_as_int(a[3]));
  }
};

struct StashSeg {
  const void *src;
  void *dst;
  int64_t n;
  int32_t block0;
};

template <int MAXSEG>
struct StashParams {
  int32_t nseg, nblocks;
  int32_t early;              // 1: start before the predecessor completes (see launch_stash_multi)
  // fused context swap: blocks [0, swap_bx * swap_n) swap, the rest stash
  const SwapEntry *swap_tab;
  int32_t swap_n, swap_bx, swap_cur, swap_next;
  StashSeg seg[MAXSEG];
};

// Context swap of table entry `entry` by block `bx` of `nbx` (see k_swap).
__device__ __forceinline__ void swap_entry(const SwapEntry *tab, int entry, int bx, int nbx, int32_t cur,
                                           int32_t next) {
  const SwapEntry e = tab[entry];
  unsigned char *live = e.live;
  unsigned char *sn = e.slot0 + (uint64_t)next * e.stride;
  unsigned char *sc = cur >= 0 ? e.slot0 + (uint64_t)cur * e.stride : nullptr;
  const uint64_t nw = e.nbytes / 16;
  const uint64_t stride = (uint64_t)nbx * blockDim.x;
  for (uint64_t w = (uint64_t)bx * blockDim.x + threadIdx.x; w < nw; w += stride) {
    // Same thread reads both copies before writing either: no save/load race.
    int4 a = reinterpret_cast<const int4 *>(live)[w];
    int4 b = reinterpret_cast<const int4 *>(sn)[w];
    if (sc) reinterpret_cast<int4 *>(sc)[w] = a;
    reinterpret_cast<int4 *>(live)[w] = b;
  }
  if (bx == 0 && threadIdx.x < e.nbytes - nw * 16) {
    const uint64_t i = nw * 16 + threadIdx.x;
    unsigned char a = live[i], b = sn[i];
    if (sc) sc[i] = a;
    live[i] = b;
  }
}

int swap_blocks_per_entry(uint64_t max_nbytes) {
  const uint64_t words = max_nbytes / 16 + 1;
  return (int)std::max<uint64_t>(1, std::min<uint64_t>((words + 255) / 256, 64));
}

// WC (warp-contiguous): a warp's kU units are 32*kU adjacent units (one
// 512*kU-byte run); otherwise a thread's kU units are a grid stride apart.
template <typename S, typename D, int E, int kU, int MAXSEG, bool WC>
__global__ void __launch_bounds__(256) k_stash(const __grid_constant__ StashParams<MAXSEG> p) {
  using In = typename VecT<S::kSize * E>::T;
  using Out = typename VecT<D::kSize * E>::T;
  if (p.early) pdl_trigger();
  else pdl_enter();
  const int nswap = p.swap_bx * p.swap_n;
  if ((int)blockIdx.x < nswap) {
    if (p.early) pdl_wait();
    swap_entry(p.swap_tab, (int)blockIdx.x / p.swap_bx, (int)blockIdx.x % p.swap_bx, p.swap_bx, p.swap_cur,
               p.swap_next);
    return;
  }
  const int bid = (int)blockIdx.x - nswap;
  const int si = find_seg(p.seg, p.nseg, bid);
  const StashSeg &g = p.seg[si];
  const int nb = (si + 1 < p.nseg ? p.seg[si + 1].block0 : p.nblocks) - g.block0;
  const In *s = reinterpret_cast<const In *>(g.src);
  Out *d = reinterpret_cast<Out *>(g.dst);
  const int64_t nunits = g.n / E;
  const int64_t stride = (int64_t)nb * blockDim.x;
  const int64_t gid = (int64_t)(bid - g.block0) * blockDim.x + threadIdx.x;
  if (WC) {
    const int lane = threadIdx.x & 31;
    const int64_t nwarps = stride >> 5;
    for (int64_t w0 = gid >> 5; w0 * 32 * kU < nunits; w0 += nwarps) {
      const int64_t base = w0 * 32 * kU + lane;
      In in[kU];
#pragma unroll
      for (int u = 0; u < kU; ++u)
        if (base + 32 * u < nunits) in[u] = ld_stream(s + base + 32 * u);
#pragma unroll
      for (int u = 0; u < kU; ++u)
        if (base + 32 * u < nunits) st_stream(d + base + 32 * u, Cast<S, D, E>::apply(in[u]));
    }
  } else {
    for (int64_t u0 = gid; u0 < nunits; u0 += stride * kU) {
      In in[kU];
#pragma unroll
      for (int u = 0; u < kU; ++u) {                      // all loads first ...
        const int64_t i = u0 + u * stride;
        if (i < nunits) in[u] = ld_stream(s + i);
      }
#pragma unroll
      for (int u = 0; u < kU; ++u) {                      // ... then the (cast and) stores
        const int64_t i = u0 + u * stride;
        if (i < nunits) st_stream(d + i, Cast<S, D, E>::apply(in[u]));
      }
    }
  }
  const int64_t tail0 = nunits * E;
  if (gid < g.n - tail0) {
    const int64_t i = tail0 + gid;
    if (S::kSize == D::kSize) {
      if (S::kSize == 4) reinterpret_cast<uint32_t *>(g.dst)[i] = reinterpret_cast<const uint32_t *>(g.src)[i];
      else reinterpret_cast<uint16_t *>(g.dst)[i] = reinterpret_cast<const uint16_t *>(g.src)[i];
    } else {
      D::store1(g.dst, i, S::load1(g.src, i));
    }
  }
  if (p.early) pdl_wait();   // complete only after the predecessor: keeps completion order transitive
}

template <typename S, typename D, int E, int kU, bool WC>
cudaError_t launch_stash_v(const StashSegDesc *segs, int nseg, cudaStream_t s, int bo, int to, int *launches,
                           const SwapArgs *swap, bool early) {
  constexpr int kMaxSeg = 32;
  const int threads = to > 0 ? to : 256;
  for (int i = 0; i < nseg; i += kMaxSeg) {
    const int k = std::min(kMaxSeg, nseg - i);
    StashParams<kMaxSeg> p;
    p.nseg = k;
    p.early = early && g_stash_early_ok && i == 0 ? 1 : 0;
    const bool fuse = i == 0 && swap && swap->n > 0;
    p.swap_tab = fuse ? swap->tab : nullptr;
    p.swap_n = fuse ? swap->n : 0;
    p.swap_bx = fuse ? swap_blocks_per_entry(swap->max_nbytes) : 0;
    p.swap_cur = fuse ? swap->cur : -1;
    p.swap_next = fuse ? swap->next : 0;
    std::vector<int64_t> work(k);
    int64_t units = 0;
    for (int j = 0; j < k; ++j) {
      p.seg[j].src = segs[i + j].src;
      p.seg[j].dst = segs[i + j].dst;
      p.seg[j].n = segs[i + j].n;
      work[j] = (segs[i + j].n + E - 1) / E;
      units += work[j];
    }
    // one-shot grid: ~one iteration of kU units per thread (profiles/r01_stash_variants.md)
    int total = (int)std::min<int64_t>((units + (int64_t)threads * kU - 1) / ((int64_t)threads * kU),
                                       (int64_t)kMaxBlocks);
    if (bo > 0) total = bo;
    else if (bo < 0) total = std::min(total, -bo);   // a cap (ES_OPT_STASH_BACKGROUND)
    total = std::max(total, k);
    std::vector<int32_t> block0;
    split_blocks(work, total, &block0, &p.nblocks);
    for (int j = 0; j < k; ++j) p.seg[j].block0 = block0[j];
    const int grid = p.nblocks + p.swap_bx * p.swap_n;
    cudaError_t e = launch_k<k_stash<S, D, E, kU, kMaxSeg, WC>>(dim3(grid), dim3(threads), s, p);
    if (e != cudaSuccess) return e;
    ++*launches;
  }
  return cudaSuccess;
}

// Stash variants were measured in round 1 (profiles/r01_stash_variants.md: unroll 1/2/8,
// cache-streaming and L2 evict-first stores, contiguous equal ranges per block in whole
// waves, TMA bulk copies) and the losers removed.  Kept: one-shot grid, 4 units in flight
// per thread; bf16 -> bf16 warp-contiguous (0.6 % faster per BERT step, 1.1421 vs 1.1496
// ms), everything else grid-stride (ResNet-50 0.3519 vs 0.3541 ms, Swin-B 4.871 vs 4.879).
template <typename S, typename D, int E>
cudaError_t launch_stash_t(const StashSegDesc *segs, int nseg, cudaStream_t s, int bo, int to, int *launches,
                           const SwapArgs *swap, bool early) {
  constexpr bool kWC = std::is_same<S, BF16T>::value && std::is_same<D, BF16T>::value;
  return launch_stash_v<S, D, E, 4, kWC>(segs, nseg, s, bo, to, launches, swap, early);
}

// ---- k_copy_tma: TMA bulk-copy stash for same-dtype segments ------------------
// One elected thread per CTA streams a contiguous, equal share of the bytes
// through an S-stage shared-memory ring: cp.async.bulk global->shared
// (completion on an mbarrier with expect_tx), then cp.async.bulk
// shared->global.  Used by ES_OPT_STASH_BACKGROUND only (S=4 x 4 KB, one warp
// per SM: a footprint that fits beside a GEMM's CTA); alone it is slower than
// k_stash (profiles/r01_stash_variants.md, r01_overlap.md).

struct CopySeg {
  const unsigned char *src;
  unsigned char *dst;
  uint64_t bytes;
};

struct CopyTmaParams {
  int32_t nseg;
  uint64_t total16;            // sum of floor16(bytes)
  uint64_t per_cta;            // multiple of 16
  CopySeg seg[32];
};

template <int S, int T>
__global__ void __launch_bounds__(32) k_copy_tma(const __grid_constant__ CopyTmaParams p) {
  extern __shared__ __align__(128) unsigned char ring[];
  __shared__ __align__(8) uint64_t bars[S];
  pdl_enter();
  if (threadIdx.x != 0) return;
  for (int st = 0; st < S; ++st)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&bars[st])) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  uint64_t pos = (uint64_t)blockIdx.x * p.per_cta;
  const uint64_t end = min(pos + p.per_cta, p.total16);
  // cursor over the concatenated floor16 space
  int si = 0;
  uint64_t seg_base = 0;
  auto next_tile = [&](const unsigned char *&src, unsigned char *&dst, uint32_t &n) -> bool {
    while (pos < end) {
      const uint64_t len = p.seg[si].bytes & ~uint64_t(15);
      if (pos >= seg_base + len) {
        seg_base += len;
        ++si;
        continue;
      }
      const uint64_t off = pos - seg_base;
      const uint64_t take = min(min((uint64_t)T, end - pos), len - off);
      src = p.seg[si].src + off;
      dst = p.seg[si].dst + off;
      n = (uint32_t)take;
      pos += take;
      return true;
    }
    return false;
  };
  const unsigned char *tsrc[S] = {};
  unsigned char *tdst[S] = {};
  uint32_t tn[S] = {};
  auto load = [&](int st) {
    const uint32_t bar = smem_addr(&bars[st]);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(tn[st]) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_addr(ring + (size_t)st * T)), "l"(tsrc[st]), "r"(tn[st]), "r"(bar)
                 : "memory");
  };
  int loaded = 0;
  for (int st = 0; st < S && next_tile(tsrc[st], tdst[st], tn[st]); ++st) {
    load(st);
    ++loaded;
  }
  for (int i = 0; i < loaded; ++i) {
    const int st = i % S;
    const uint32_t bar = smem_addr(&bars[st]);
    const uint32_t parity = (uint32_t)((i / S) & 1);
    uint32_t ok = 0;
    do {
      asm volatile("{\n .reg .pred q;\n mbarrier.try_wait.parity.shared::cta.b64 q, [%1], %2;\n selp.u32 %0, 1, 0, q;\n}"
                   : "=r"(ok)
                   : "r"(bar), "r"(parity)
                   : "memory");
    } while (!ok);
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(tdst[st]),
                 "r"(smem_addr(ring + (size_t)st * T)), "r"(tn[st])
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    // Refill the stage of the PREVIOUS tile: its store group is the second
    // most recent, so wait_group.read 1 returns once it has read the stage,
    // while this tile's store still runs (no load <-> store serialisation).
    if (i >= 1) {
      const int ps = (i - 1) % S;
      const unsigned char *ns;
      unsigned char *nd;
      uint32_t nn;
      if (next_tile(ns, nd, nn)) {
        asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        tsrc[ps] = ns;
        tdst[ps] = nd;
        tn[ps] = nn;
        load(ps);
        ++loaded;
      }
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  // sub-16-byte tails of the segments: CTA (segment index % grid)
  for (int k = 0; k < p.nseg; ++k) {
    if ((uint32_t)k % gridDim.x != blockIdx.x) continue;
    const uint64_t len = p.seg[k].bytes & ~uint64_t(15);
    for (uint64_t b = len; b < p.seg[k].bytes; ++b) p.seg[k].dst[b] = p.seg[k].src[b];
  }
}

template <int S, int T>
cudaError_t launch_copy_tma(const StashSegDesc *segs, int nseg, int esize, cudaStream_t s, int ctas_per_sm,
                            int *launches) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_copy_tma<S, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, S * T);
    attr = true;
  }
  for (int i = 0; i < nseg; i += 32) {
    const int k = std::min(32, nseg - i);
    CopyTmaParams p;
    p.nseg = k;
    p.total16 = 0;
    for (int j = 0; j < k; ++j) {
      p.seg[j].src = reinterpret_cast<const unsigned char *>(segs[i + j].src);
      p.seg[j].dst = reinterpret_cast<unsigned char *>(segs[i + j].dst);
      p.seg[j].bytes = (uint64_t)segs[i + j].n * esize;
      p.total16 += p.seg[j].bytes & ~uint64_t(15);
    }
    const int grid = kSMs * ctas_per_sm;
    p.per_cta = ((p.total16 + grid - 1) / grid + 15) & ~uint64_t(15);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(32);
    cfg.dynamicSmemBytes = S * T;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = g_pdl ? 1 : 0;
    (void)KernelReg<k_copy_tma<S, T>>::token;
    cudaError_t e = cudaLaunchKernelEx(&cfg, k_copy_tma<S, T>, p);
    if (e != cudaSuccess) return e;
    ++*launches;
  }
  return cudaSuccess;
}


// ---- k_swap -----------------------------------------------------------------

struct SwapParams {
  const SwapEntry *tab;
  int32_t cur, next;
};

__global__ void __launch_bounds__(256) k_swap(const __grid_constant__ SwapParams p) {
  pdl_enter();
  swap_entry(p.tab, (int)blockIdx.y, (int)blockIdx.x, (int)gridDim.x, p.cur, p.next);
}

// ---- k_dropout (NEXT-4) ------------------------------------------------------
// Philox4x32-10 (Salmon et al., SC'11) -- element i: key = seed, counter =
// (i/4, offset); word i % 4; u = (w >> 8) * 2^-24; keep = u >= p.

__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
  const uint32_t M0 = 0xD2511F53u, M1 = 0xCD9E8D57u, W0 = 0x9E3779B9u, W1 = 0xBB67AE85u;
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    if (r > 0) {
      k.x += W0;
      k.y += W1;
    }
    const uint32_t hi0 = __umulhi(M0, c.x), lo0 = M0 * c.x;
    const uint32_t hi1 = __umulhi(M1, c.z), lo1 = M1 * c.z;
    c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
  }
  return c;
}

struct DropoutParams {
  const void *x;
  void *y;
  uint8_t *mask;
  int64_t n;
  float p, scale;
  uint64_t *record;
  unsigned int *counter;
};

template <typename T>
__global__ void __launch_bounds__(256) k_dropout(const __grid_constant__ DropoutParams p) {
  pdl_enter();
  const uint64_t seed = p.record[0], offset = p.record[1];
  const uint2 key = make_uint2((uint32_t)seed, (uint32_t)(seed >> 32));
  const int64_t nq = (p.n + 3) / 4;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < nq; q += stride) {
    const uint4 w = philox4x32_10(
        make_uint4((uint32_t)q, (uint32_t)((uint64_t)q >> 32), (uint32_t)offset, (uint32_t)(offset >> 32)), key);
    const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int64_t i = q * 4 + e;
      if (i < p.n) {
        const float u = __uint2float_rn(ws[e] >> 8) * (1.0f / 16777216.0f);   // exact: 24-bit integer
        const bool keep = u >= p.p;
        T::store1(p.y, i, keep ? __fmul_rn(T::load1(p.x, i), p.scale) : 0.0f);
        if (p.mask) p.mask[i] = keep ? 1 : 0;
      }
    }
  }
  // Advance the EST's Philox offset once every block has read it.
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(p.counter, 1u) == gridDim.x - 1) {
      p.record[1] = offset + 1;
      *p.counter = 0;
      __threadfence();
    }
  }
}

// ---- k_peer_barrier (ES_SCHED_PEER) -------------------------------------------

struct BarrierParams {
  uint64_t *peer_flags[64];
  uint64_t *my_flags;
  int32_t G, rank;
  uint64_t timeout_ns;
};

__global__ void __launch_bounds__(64) k_peer_barrier(const __grid_constant__ BarrierParams p) {
  // Wait for the predecessor, but let the successor's CTAs become resident
  // only after the barrier has passed: waiting CTAs must never occupy SM
  // slots other ranks need to reach this barrier (they share a GPU under the
  // loopback transport).
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const int t = threadIdx.x;
  // Every rank runs the same sequence of barriers, so the device-resident
  // counters advance in lockstep, eager or replayed from a CUDA graph.
  const uint64_t epoch = p.my_flags[kEpochSlot] + 1;
  __threadfence_system();                       // this GPU's completed writes before the arrival
  if (t < p.G) {
    uint64_t *dst = p.peer_flags[t] + p.rank;
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(dst), "l"(epoch) : "memory");
  }
  if (t < p.G) {
    const uint64_t *src = p.my_flags + t;
    uint64_t v = 0, t0 = 0, now = 0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    do {
      asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(src) : "memory");
      if (v >= epoch) break;
      __nanosleep(256);
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
      if (now - t0 > p.timeout_ns) __trap();   // a peer never arrived: fail loudly, never hang the GPU
    } while (true);
  }
  __syncthreads();
  if (t == 0) p.my_flags[kEpochSlot] = epoch;   // read back only by this rank's next barrier
  __threadfence_system();
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

}  // namespace

void set_pdl(bool on) { g_pdl = on; }

cudaError_t preload_kernels() {
  for (const void *f : kernel_registry()) {
    cudaFuncAttributes a;
    cudaError_t e = cudaFuncGetAttributes(&a, f);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

size_t registered_kernels() { return kernel_registry().size(); }

cudaError_t launch_fold_multi(es_dtype dtype, int32_t N, float r, uint32_t compat, const FoldSegDesc *segs, int nseg,
                              cudaStream_t s, int blocks_override, int threads_override, int *launches) {
  if (dtype != ES_BF16) compat &= ~kBf16Hop;   // bf16 storage rounding only exists for bf16 buckets
  int dummy = 0;
  if (!launches) launches = &dummy;
  std::vector<FoldSegDesc> live;
  live.reserve(nseg);
  for (int i = 0; i < nseg; ++i)
    if (segs[i].n > 0) live.push_back(segs[i]);
  if (live.empty()) return cudaSuccess;
  if (dtype == ES_BF16)
    return launch_fold_t<BF16T>(N, r, compat, live.data(), (int)live.size(), s, blocks_override, threads_override,
                                launches);
  // small fp32 folds: 8 elements per thread (F32WT) when every pointer allows 32-byte accesses
  int64_t elems = 0;
  bool wide = compat == 0 && blocks_override <= 0;
  auto a32 = [](const void *q) { return (reinterpret_cast<uintptr_t>(q) & 31) == 0; };
  for (const FoldSegDesc &d : live) {
    elems += d.n;
    wide = wide && a32(d.out) && (!d.part_in || a32(d.part_in));
    for (int j = 0; wide && j < (d.rot ? N : d.m) + d.npush; ++j) wide = a32(d.src[j]);
  }
  if (wide && elems <= kWideMaxElems)
    return launch_fold_t<F32WT>(N, r, compat, live.data(), (int)live.size(), s, blocks_override, threads_override,
                                launches);
  return launch_fold_t<F32T>(N, r, compat, live.data(), (int)live.size(), s, blocks_override, threads_override,
                             launches);
}


cudaError_t launch_stash_multi(es_dtype sdt, es_dtype ddt, const StashSegDesc *segs, int nseg, cudaStream_t s,
                               int bo, int to, int *launches, const SwapArgs *swap, bool early, bool background) {
  int dummy = 0;
  if (!launches) launches = &dummy;
  std::vector<StashSegDesc> live;
  for (int i = 0; i < nseg; ++i)
    if (segs[i].n > 0) live.push_back(segs[i]);
  if (live.empty()) {
    if (swap && swap->n > 0) {
      ++*launches;
      return launch_swap(swap->tab, swap->n, swap->max_nbytes, swap->cur, swap->next, s);
    }
    return cudaSuccess;
  }
  const int n = (int)live.size();
  bool aligned = true;
  for (const StashSegDesc &g : live)
    aligned = aligned && !(reinterpret_cast<uintptr_t>(g.src) & 15) && !(reinterpret_cast<uintptr_t>(g.dst) & 15);
  if (background && sdt == ddt && aligned && bo <= 0) {   // bo > 0: an explicit es_set_launch_override
    // ES_OPT_STASH_BACKGROUND, same dtype: the copy runs as one warp per SM
    // driving a 4 x 4 KB TMA bulk-copy ring (16 KB of shared memory, a
    // few registers), a footprint that fits beside a tensor-core GEMM's CTA, so
    // the stash streams while the model computes (profiles/r01_overlap.md).
    // The context swap, if any, is its own small launch first.
    if (swap && swap->n > 0) {
      ++*launches;
      cudaError_t e = launch_swap(swap->tab, swap->n, swap->max_nbytes, swap->cur, swap->next, s);
      if (e != cudaSuccess) return e;
    }
    return launch_copy_tma<4, 4096>(live.data(), n, sdt == ES_BF16 ? 2 : 4, s, 1, launches);
  }
  if (sdt == ES_F32 && ddt == ES_F32) return launch_stash_t<F32T, F32T, 4>(live.data(), n, s, bo, to, launches, swap, early);
  if (sdt == ES_BF16 && ddt == ES_BF16)
    return launch_stash_t<BF16T, BF16T, 8>(live.data(), n, s, bo, to, launches, swap, early);
  if (sdt == ES_F32 && ddt == ES_BF16)
    return launch_stash_t<F32T, BF16T, 4>(live.data(), n, s, bo, to, launches, swap, early);
  return launch_stash_t<BF16T, F32T, 4>(live.data(), n, s, bo, to, launches, swap, early);
}

cudaError_t launch_fold_pipe(es_dtype dtype, int32_t N, float r, const PipeSegDesc *segs, int nseg,
                             const uint64_t *epoch, unsigned int *ticket, int share, cudaStream_t s, int *launches) {
  int dummy = 0;
  if (!launches) launches = &dummy;
  std::vector<PipeSegDesc> live;
  for (int i = 0; i < nseg; ++i)
    if (segs[i].f.n > 0) live.push_back(segs[i]);
  if (live.empty()) return cudaSuccess;
  if (dtype == ES_BF16)
    return launch_pipe_t<BF16T>(N, r, live.data(), (int)live.size(), epoch, ticket, share, s, launches);
  return launch_pipe_t<F32T>(N, r, live.data(), (int)live.size(), epoch, ticket, share, s, launches);
}

cudaError_t launch_dropout(es_dtype dtype, const void *x, void *y, uint8_t *mask, int64_t n, float p, float scale,
                           uint64_t *record, unsigned int *counter, cudaStream_t s) {
  DropoutParams d{x, y, mask, n, p, scale, record, counter};
  const int64_t nq = std::max<int64_t>((n + 3) / 4, 1);
  const int blocks = (int)std::min<int64_t>((nq + 255) / 256, (int64_t)kSMs * 16);
  if (dtype == ES_BF16) return launch_k<k_dropout<BF16T>>(dim3(blocks), dim3(256), s, d);
  return launch_k<k_dropout<F32T>>(dim3(blocks), dim3(256), s, d);
}

cudaError_t launch_peer_barrier(uint64_t *const *peer_flags, uint64_t *my_flags, int32_t G, int32_t rank,
                                cudaStream_t s) {
  if (G < 1 || G > 64) return cudaErrorInvalidValue;
  BarrierParams b;
  for (int i = 0; i < 64; ++i) b.peer_flags[i] = i < G ? peer_flags[i] : nullptr;
  b.my_flags = my_flags;
  b.G = G;
  b.rank = rank;
  b.timeout_ns = barrier_timeout_ns();
  return launch_k<k_peer_barrier>(dim3(1), dim3(64), s, b);
}

cudaError_t launch_swap(const SwapEntry *table_dev, int32_t n, uint64_t max_nbytes, int32_t cur, int32_t next,
                        cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  SwapParams p{table_dev, cur, next};
  return launch_k<k_swap>(dim3(swap_blocks_per_entry(max_nbytes), (unsigned)n), dim3(256), s, p);
}

}  // namespace es
