// kernels.cu -- the sm_100a kernels of libes.
//
//   k_fold  : canonical-order fold + fused 1/N post-scale
//   k_stash : vectorised copy / cast into an EST's slot       (8(a) a1)
//   k_swap  : context-switch save/load of per-EST state       (8(a) a2)
//
// All three are HBM-streaming kernels (no data reuse, no contraction), so
// they use 128-bit vector loads on the non-coherent path with L1
// no-allocate, many independent loads in flight per thread, and grids sized
// in multiples of the 148 SMs.
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

namespace es {
namespace {

constexpr int kSMs = 148;        // B200
constexpr int kBatch = 8;        // sources loaded per batch in k_fold

__device__ __forceinline__ int4 ld_stream(const void *p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ void st_stream(void *p, const int4 &v) {
  asm volatile("st.global.L1::no_allocate.v4.s32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y),
               "r"(v.z), "r"(v.w)
               : "memory");
}

// ---- element-type traits --------------------------------------------------
// A "vector" is 16 bytes of the bucket dtype: 4 fp32 or 8 bf16.

struct F32T {
  static constexpr int kVec = 4;
  static constexpr int kSize = 4;
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
  // bf16 is the high half of an fp32: widening is exact (R4).
  __device__ static __forceinline__ void widen2(uint32_t w, float *a) {
    a[0] = __uint_as_float(w << 16);
    a[1] = __uint_as_float(w & 0xFFFF0000u);
  }
  __device__ static __forceinline__ void widen(const int4 &v, float *a) {
    widen2((uint32_t)v.x, a + 0); widen2((uint32_t)v.y, a + 2);
    widen2((uint32_t)v.z, a + 4); widen2((uint32_t)v.w, a + 6);
  }
  __device__ static __forceinline__ uint32_t pack2(float lo, float hi) {
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

// ---- k_fold ---------------------------------------------------------------

template <int MAXN>
struct FoldParams {
  const void *src[MAXN];
  const float *part_in;
  void *out;
  int64_t lo;
  int64_t n;
  int32_t N;
  int32_t m;
  uint32_t C;
  int32_t rot;
  int32_t out_partial;
  float r;
};

template <typename T, int MAXN>
__device__ __forceinline__ void fold_vector(const FoldParams<MAXN> &p, int64_t t, float *acc) {
  constexpr int V = T::kVec;
  int cnt, idx;
  if (p.rot) {
    const uint32_t c = (uint32_t)(p.lo + t) / p.C;          // R1: chunk of this vector
    idx = (int)(c + 1u == (uint32_t)p.N ? 0u : c + 1u);      // R2: start at rank c+1
    cnt = p.N;
  } else {
    idx = 0;
    cnt = p.m;
  }
  const int64_t boff = t * T::kSize;                         // byte offset of the vector
  int done = 0;
  if (p.part_in) {                                           // continue a chain partial
    const float *pp = p.part_in + t;
#pragma unroll
    for (int q = 0; q < V / 4; ++q) {
      int4 w = ld_stream(pp + 4 * q);
      acc[4 * q + 0] = __int_as_float(w.x); acc[4 * q + 1] = __int_as_float(w.y);
      acc[4 * q + 2] = __int_as_float(w.z); acc[4 * q + 3] = __int_as_float(w.w);
    }
  } else {                                                   // R3: start from the first contribution
    int4 w = ld_stream(reinterpret_cast<const char *>(p.src[idx]) + boff);
    T::widen(w, acc);
    idx = (idx + 1 == cnt) ? 0 : idx + 1;
    done = 1;
  }
  while (done < cnt) {
    const int nb = min(kBatch, cnt - done);
    int4 buf[kBatch];
    int k = idx;
#pragma unroll
    for (int b = 0; b < kBatch; ++b) {                       // all loads of the batch first ...
      if (b < nb) {
        buf[b] = ld_stream(reinterpret_cast<const char *>(p.src[k]) + boff);
        k = (k + 1 == cnt) ? 0 : k + 1;
      }
    }
#pragma unroll
    for (int b = 0; b < kBatch; ++b) {                       // ... then the adds, in canonical order
      if (b < nb) {
        float x[V];
        T::widen(buf[b], x);
#pragma unroll
        for (int e = 0; e < V; ++e) acc[e] = __fadd_rn(acc[e], x[e]);
      }
    }
    idx = k;
    done += nb;
  }
}

template <typename T, int MAXN>
__device__ __forceinline__ float fold_scalar(const FoldParams<MAXN> &p, int64_t t) {
  int cnt, idx;
  if (p.rot) {
    const uint32_t c = (uint32_t)(p.lo + t) / p.C;
    idx = (int)(c + 1u == (uint32_t)p.N ? 0u : c + 1u);
    cnt = p.N;
  } else {
    idx = 0;
    cnt = p.m;
  }
  float s;
  int done = 0;
  if (p.part_in) {
    s = p.part_in[t];
  } else {
    s = T::load1(p.src[idx], t);
    idx = (idx + 1 == cnt) ? 0 : idx + 1;
    done = 1;
  }
  for (; done < cnt; ++done) {
    s = __fadd_rn(s, T::load1(p.src[idx], t));
    idx = (idx + 1 == cnt) ? 0 : idx + 1;
  }
  return s;
}

template <typename T, int MAXN>
__global__ void __launch_bounds__(256) k_fold(const __grid_constant__ FoldParams<MAXN> p) {
  constexpr int V = T::kVec;
  const int64_t nvec = p.n / V;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (int64_t v = gid; v < nvec; v += stride) {
    const int64_t t = v * V;
    float acc[V];
    fold_vector<T, MAXN>(p, t, acc);
    if (p.out_partial) {
      float *o = reinterpret_cast<float *>(p.out) + t;
#pragma unroll
      for (int q = 0; q < V / 4; ++q)
        st_stream(o + 4 * q, make_int4(__float_as_int(acc[4 * q]), __float_as_int(acc[4 * q + 1]),
                                       __float_as_int(acc[4 * q + 2]), __float_as_int(acc[4 * q + 3])));
    } else {
#pragma unroll
      for (int e = 0; e < V; ++e) acc[e] = __fmul_rn(acc[e], p.r);   // R5: one rounding
      st_stream(reinterpret_cast<char *>(p.out) + t * T::kSize, T::narrow(acc));  // R13
    }
  }
  // Ragged tail (< V elements).
  const int64_t tail0 = nvec * V;
  if (gid < p.n - tail0) {
    const int64_t t = tail0 + gid;
    float s = fold_scalar<T, MAXN>(p, t);
    if (p.out_partial) reinterpret_cast<float *>(p.out)[t] = s;
    else T::store1(p.out, t, __fmul_rn(s, p.r));
  }
}

template <typename T, int MAXN>
cudaError_t launch_fold_t(const FoldDesc &d, const void *const *src, cudaStream_t s, int bo, int to) {
  FoldParams<MAXN> p;
  const int nsrc = d.rot ? d.N : d.m;
  for (int j = 0; j < nsrc; ++j) p.src[j] = src[j];
  for (int j = nsrc; j < MAXN; ++j) p.src[j] = nullptr;
  p.part_in = d.part_in;
  p.out = d.out;
  p.lo = d.lo;
  p.n = d.n;
  p.N = d.N;
  p.m = d.m;
  p.C = d.C;
  p.rot = d.rot ? 1 : 0;
  p.out_partial = d.out_partial ? 1 : 0;
  p.r = d.r;
  const int threads = to > 0 ? to : 256;
  const int64_t nvec = d.n / T::kVec;
  int64_t want = (std::max<int64_t>(nvec, 1) + threads - 1) / threads;
  int blocks = (int)std::min<int64_t>(want, (int64_t)kSMs * 8);
  if (bo > 0) blocks = bo;
  k_fold<T, MAXN><<<blocks, threads, 0, s>>>(p);
  return cudaGetLastError();
}

template <typename T>
cudaError_t launch_fold_dt(const FoldDesc &d, const void *const *src, cudaStream_t s, int bo, int to) {
  const int nsrc = d.rot ? d.N : d.m;
  if (nsrc <= 8) return launch_fold_t<T, 8>(d, src, s, bo, to);
  if (nsrc <= 32) return launch_fold_t<T, 32>(d, src, s, bo, to);
  if (nsrc <= 128) return launch_fold_t<T, 128>(d, src, s, bo, to);
  return launch_fold_t<T, 1024>(d, src, s, bo, to);
}

// ---- k_stash ----------------------------------------------------------------
// Groups of 8 elements: fp32 = 2 vectors, bf16 = 1 vector.  kU groups per
// thread per iteration, all loads issued before the stores.

template <typename S, typename D, int kU>
__global__ void __launch_bounds__(256) k_stash(const void *__restrict__ src, void *__restrict__ dst, int64_t n) {
  constexpr int kInVec = S::kSize * 8 / 16;    // 16-byte loads per group
  constexpr int kOutVec = D::kSize * 8 / 16;   // 16-byte stores per group
  const int64_t ngroups = n / 8;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const char *s8 = reinterpret_cast<const char *>(src);
  char *d8 = reinterpret_cast<char *>(dst);
  for (int64_t g0 = gid; g0 < ngroups; g0 += stride * kU) {
    int4 in[kU][kInVec];
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const int64_t g = g0 + u * stride;
      if (g < ngroups) {
#pragma unroll
        for (int q = 0; q < kInVec; ++q) in[u][q] = ld_stream(s8 + g * 8 * S::kSize + q * 16);
      }
    }
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const int64_t g = g0 + u * stride;
      if (g < ngroups) {
        if (S::kSize == D::kSize) {
#pragma unroll
          for (int q = 0; q < kInVec; ++q) st_stream(d8 + g * 8 * D::kSize + q * 16, in[u][q]);
        } else {
          float a[8];
#pragma unroll
          for (int q = 0; q < kInVec; ++q) S::widen(in[u][q], a + q * S::kVec);
#pragma unroll
          for (int q = 0; q < kOutVec; ++q) st_stream(d8 + g * 8 * D::kSize + q * 16, D::narrow(a + q * D::kVec));
        }
      }
    }
  }
  const int64_t tail0 = ngroups * 8;
  if (gid < n - tail0) {
    const int64_t i = tail0 + gid;
    if (S::kSize == D::kSize) {
      if (S::kSize == 4) reinterpret_cast<uint32_t *>(dst)[i] = reinterpret_cast<const uint32_t *>(src)[i];
      else reinterpret_cast<uint16_t *>(dst)[i] = reinterpret_cast<const uint16_t *>(src)[i];
    } else {
      D::store1(dst, i, S::load1(src, i));
    }
  }
}

template <typename S, typename D>
cudaError_t launch_stash_t(const void *src, void *dst, int64_t n, cudaStream_t s, int bo, int to) {
  constexpr int kU = 4;
  const int threads = to > 0 ? to : 256;
  const int64_t groups = std::max<int64_t>(n / 8, 1);
  int64_t want = (groups + (int64_t)threads * kU - 1) / ((int64_t)threads * kU);
  int blocks = (int)std::min<int64_t>(std::max<int64_t>(want, 1), (int64_t)kSMs * 8);
  if (bo > 0) blocks = bo;
  k_stash<S, D, kU><<<blocks, threads, 0, s>>>(src, dst, n);
  return cudaGetLastError();
}

// ---- k_swap -----------------------------------------------------------------

__global__ void __launch_bounds__(256) k_swap(const SwapEntry *__restrict__ tab, int32_t cur, int32_t next) {
  const SwapEntry e = tab[blockIdx.y];
  unsigned char *live = e.live;
  unsigned char *sn = e.slot0 + (uint64_t)next * e.stride;
  unsigned char *sc = cur >= 0 ? e.slot0 + (uint64_t)cur * e.stride : nullptr;
  const uint64_t nw = e.nbytes / 16;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += stride) {
    // Same thread reads both copies before writing either: no save/load race.
    int4 a = reinterpret_cast<const int4 *>(live)[w];
    int4 b = reinterpret_cast<const int4 *>(sn)[w];
    if (sc) reinterpret_cast<int4 *>(sc)[w] = a;
    reinterpret_cast<int4 *>(live)[w] = b;
  }
  if (blockIdx.x == 0 && threadIdx.x < e.nbytes - nw * 16) {
    const uint64_t i = nw * 16 + threadIdx.x;
    unsigned char a = live[i], b = sn[i];
    if (sc) sc[i] = a;
    live[i] = b;
  }
}

}  // namespace

cudaError_t launch_fold(es_dtype dtype, const FoldDesc &d, const void *const *src, cudaStream_t s,
                        int blocks_override, int threads_override) {
  if (d.n <= 0) return cudaSuccess;
  if (dtype == ES_BF16) return launch_fold_dt<BF16T>(d, src, s, blocks_override, threads_override);
  return launch_fold_dt<F32T>(d, src, s, blocks_override, threads_override);
}

cudaError_t launch_stash(const void *src, es_dtype sdt, void *dst, es_dtype ddt, int64_t n, cudaStream_t s,
                         int bo, int to) {
  if (n <= 0) return cudaSuccess;
  if (sdt == ES_F32 && ddt == ES_F32) return launch_stash_t<F32T, F32T>(src, dst, n, s, bo, to);
  if (sdt == ES_BF16 && ddt == ES_BF16) return launch_stash_t<BF16T, BF16T>(src, dst, n, s, bo, to);
  if (sdt == ES_F32 && ddt == ES_BF16) return launch_stash_t<F32T, BF16T>(src, dst, n, s, bo, to);
  return launch_stash_t<BF16T, F32T>(src, dst, n, s, bo, to);
}

cudaError_t launch_swap(const SwapEntry *table_dev, int32_t n, uint64_t max_nbytes, int32_t cur, int32_t next,
                        cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  uint64_t words = max_nbytes / 16 + 1;
  int bx = (int)std::min<uint64_t>((words + 255) / 256, 64);
  dim3 grid(std::max(bx, 1), (unsigned)n);
  k_swap<<<grid, 256, 0, s>>>(table_dev, cur, next);
  return cudaGetLastError();
}

}  // namespace es
