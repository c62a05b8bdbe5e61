// probe_read.cu -- HBM ceiling probes for the fold's access pattern (not product code).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/probe_read scripts/probe_read.cu
//   ./probe_read            (one GPU; prints one JSON line per variant)
//
// (1) read-only stream of one buffer (sum, one tiny write per block): the pure-read ceiling;
// (2) copy (read + write, the MEASURED_PEAKS definition);
// (3) the fold's pattern: N sources read at the same offset, one result written per element
//     (N/(N+1) reads), with U consecutive 16-B vectors per thread per source (U = 1 is k_fold's
//     current shape) -- does more contiguous bytes per source and warp help the DRAM row buffers?
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s\n", cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ int4 ldnc(const void *p) {
  int4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ void stna(void *p, int4 v) {
  asm volatile("st.global.L1::no_allocate.v4.s32 [%0], {%1,%2,%3,%4};" :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w));
}

__global__ void k_read(const int4 *a, int64_t nvec, int *sink) {
  int acc = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvec; i += (int64_t)gridDim.x * blockDim.x * 4) {
    int4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      int64_t j = i + (int64_t)u * gridDim.x * blockDim.x;
      v[u] = j < nvec ? ldnc(a + j) : make_int4(0, 0, 0, 0);
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  if (acc == 0x12345678) sink[blockIdx.x] = acc;
}

__global__ void k_copy(const int4 *a, int4 *b, int64_t nvec) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvec; i += (int64_t)gridDim.x * blockDim.x * 4) {
    int4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      int64_t j = i + (int64_t)u * gridDim.x * blockDim.x;
      if (j < nvec) v[u] = ldnc(a + j);
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      int64_t j = i + (int64_t)u * gridDim.x * blockDim.x;
      if (j < nvec) stna(b + j, v[u]);
    }
  }
}

// one-shot read: every thread loads 4 vectors (warp-contiguous), no grid-stride loop
__global__ void __launch_bounds__(256) k_read1(const int4 *a, int64_t nvec, int *sink) {
  const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t base = w * 128 + lane;
  int4 v[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) v[u] = ldnc(a + base + 32 * u);
  int acc = 0;
#pragma unroll
  for (int u = 0; u < 4; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  if (acc == 0x12345678) sink[blockIdx.x & 1023] = acc;
}

// one-shot copy: every thread moves U warp-contiguous 16-B vectors (all loads, then all stores)
template <int U>
__global__ void __launch_bounds__(256) k_copy1(const int4 *a, int4 *b, int64_t nvec) {
  const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t base = w * 32 * U + lane;
  int4 v[U];
#pragma unroll
  for (int u = 0; u < U; ++u)
    if (base + 32 * u < nvec) v[u] = ldnc(a + base + 32 * u);
#pragma unroll
  for (int u = 0; u < U; ++u)
    if (base + 32 * u < nvec) stna(b + base + 32 * u, v[u]);
}

// k_stash's current pattern: one-shot grid, U units per thread at grid-wide stride
template <int U>
__global__ void __launch_bounds__(256) k_copy_gs(const int4 *a, int4 *b, int64_t nvec) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (int64_t u0 = g; u0 < nvec; u0 += stride * U) {
    int4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (u0 + u * stride < nvec) v[u] = ldnc(a + u0 + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (u0 + u * stride < nvec) stna(b + u0 + u * stride, v[u]);
  }
}

struct Srcs { const float *p[32]; };

// fold pattern: element-vector v of every source; U consecutive vectors per thread (warp covers
// 32*U*16 contiguous bytes of each source), sources in batches of 8.
template <int U, bool WRITE = true>
__global__ void __launch_bounds__(256) k_foldpat(const __grid_constant__ Srcs s, int N, float *out, int64_t nvec) {
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t w = warp; w * 32 * U < nvec; w += nwarps) {
    float acc[U][4];
    const int64_t base = w * 32 * U + lane;
#pragma unroll
    for (int u = 0; u < U; ++u) acc[u][0] = acc[u][1] = acc[u][2] = acc[u][3] = 0.f;
    for (int k0 = 0; k0 < N; k0 += 8) {
      int4 buf[8][U];
#pragma unroll
      for (int b = 0; b < 8; ++b)
#pragma unroll
        for (int u = 0; u < U; ++u) {
          int64_t j = base + 32 * u;
          if (k0 + b < N && j < nvec) buf[b][u] = ldnc(reinterpret_cast<const int4 *>(s.p[k0 + b]) + j);
          else buf[b][u] = make_int4(0, 0, 0, 0);
        }
#pragma unroll
      for (int b = 0; b < 8; ++b)
#pragma unroll
        for (int u = 0; u < U; ++u) {
          acc[u][0] = __fadd_rn(acc[u][0], __int_as_float(buf[b][u].x));
          acc[u][1] = __fadd_rn(acc[u][1], __int_as_float(buf[b][u].y));
          acc[u][2] = __fadd_rn(acc[u][2], __int_as_float(buf[b][u].z));
          acc[u][3] = __fadd_rn(acc[u][3], __int_as_float(buf[b][u].w));
        }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      int64_t j = base + 32 * u;
      if (j < nvec && (WRITE || acc[u][0] == 1234.5f))
        stna(reinterpret_cast<int4 *>(out) + j, make_int4(__float_as_int(acc[u][0]), __float_as_int(acc[u][1]),
                                                         __float_as_int(acc[u][2]), __float_as_int(acc[u][3])));
    }
  }
}

// bf16 fold pattern (BERT: N = 12): 8 bf16 per 16-B vector widened to fp32, folded, rounded back;
// sources loaded in batches of BATCH (k_fold uses 8: 8 + 4 for N = 12).
template <int BATCH>
__global__ void __launch_bounds__(256) k_foldpat_bf16(const __grid_constant__ Srcs s, int N, uint16_t *out,
                                                     int64_t nvec) {
  const int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v >= nvec) return;
  float acc[8];
#pragma unroll
  for (int e = 0; e < 8; ++e) acc[e] = 0.f;
  for (int k0 = 0; k0 < N; k0 += BATCH) {
    int4 buf[BATCH];
#pragma unroll
    for (int b = 0; b < BATCH; ++b)
      buf[b] = k0 + b < N ? ldnc(reinterpret_cast<const int4 *>(s.p[k0 + b]) + v) : make_int4(0, 0, 0, 0);
#pragma unroll
    for (int b = 0; b < BATCH; ++b) {
      if (k0 + b < N) {
        const uint32_t w[4] = {(uint32_t)buf[b].x, (uint32_t)buf[b].y, (uint32_t)buf[b].z, (uint32_t)buf[b].w};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          acc[2 * q] = __fadd_rn(acc[2 * q], __uint_as_float(w[q] << 16));
          acc[2 * q + 1] = __fadd_rn(acc[2 * q + 1], __uint_as_float(w[q] & 0xffff0000u));
        }
      }
    }
  }
  uint32_t o[4];
#pragma unroll
  for (int q = 0; q < 4; ++q)
    o[q] = (__float_as_uint(acc[2 * q]) >> 16) | (__float_as_uint(acc[2 * q + 1]) & 0xffff0000u);
  stna(reinterpret_cast<int4 *>(out) + v, make_int4(o[0], o[1], o[2], o[3]));
}

template <typename F>
static float best_ms(F f, int reps = 10) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  float best = 1e30f;
  for (int r = 0; r < reps + 2; ++r) {
    cudaEventRecord(a);
    f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    if (r >= 2 && ms < best) best = ms;
  }
  return best;
}

int main() {
  const int64_t bytes = 4ll << 30;                 // 4 GiB read stream
  const int64_t nvec = bytes / 16;
  char *a, *b; int *sink;
  CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes)); CK(cudaMalloc(&sink, 1 << 20));
  CK(cudaMemset(a, 1, bytes)); CK(cudaMemset(b, 0, bytes));
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int g : {sms * 4, sms * 8, sms * 16, sms * 32}) {
    float ms = best_ms([&] { k_read<<<g, 256>>>((const int4 *)a, nvec, sink); });
    printf("{\"probe\": \"read\", \"grid\": %d, \"GBps\": %.1f}\n", g, bytes / (ms * 1e-3) / 1e9);
  }
  {
    const int g = (int)(nvec / (256 * 4));
    float ms = best_ms([&] { k_read1<<<g, 256>>>((const int4 *)a, nvec, sink); });
    printf("{\"probe\": \"read_oneshot\", \"grid\": %d, \"GBps\": %.1f}\n", g, bytes / (ms * 1e-3) / 1e9);
  }
  for (int g : {sms * 4, sms * 8, sms * 16}) {
    float ms = best_ms([&] { k_copy<<<g, 256>>>((const int4 *)a, (int4 *)b, nvec / 2); });
    printf("{\"probe\": \"copy\", \"grid\": %d, \"GBps\": %.1f}\n", g, bytes / (ms * 1e-3) / 1e9);
  }
  {  // one-shot copies of 2 GiB (read + write bytes counted), U vectors per thread
    const int64_t nv = nvec / 2;
    float m1 = best_ms([&] { k_copy1<1><<<(int)((nv + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, nv); });
    float m2 = best_ms([&] { k_copy1<2><<<(int)((nv / 2 + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, nv); });
    float m4 = best_ms([&] { k_copy1<4><<<(int)((nv / 4 + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, nv); });
    float m8 = best_ms([&] { k_copy1<8><<<(int)((nv / 8 + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, nv); });
    float mc = best_ms([&] { cudaMemcpyAsync(b, a, bytes / 2, cudaMemcpyDeviceToDevice); });
    float g4 = best_ms([&] { k_copy_gs<4><<<(int)((nv / 4 + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, nv); });
    float g2 = best_ms([&] { k_copy_gs<2><<<(int)((nv / 2 + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, nv); });
    // ResNet-50-sized stash: 102 MB one way (L2 = 126 MB)
    const int64_t ns = 25557032 / 4;
    float s4 = best_ms([&] { k_copy_gs<4><<<(int)((ns / 4 + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, ns); });
    float s2w = best_ms([&] { k_copy1<2><<<(int)((ns / 2 + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, ns); });
    float s4w = best_ms([&] { k_copy1<4><<<(int)((ns / 4 + 255) / 256), 256>>>((const int4 *)a, (int4 *)b, ns); });
    printf("{\"probe\": \"copy_gridstride_oneshot\", \"U4_GBps\": %.1f, \"U2_GBps\": %.1f, "
           "\"resnet_stash_102MB\": {\"gridstride_U4\": %.1f, \"warp_U2\": %.1f, \"warp_U4\": %.1f}}\n",
           bytes / (g4 * 1e-3) / 1e9, bytes / (g2 * 1e-3) / 1e9, 32.0 * ns / (s4 * 1e-3) / 1e9,
           32.0 * ns / (s2w * 1e-3) / 1e9, 32.0 * ns / (s4w * 1e-3) / 1e9);
    printf("{\"probe\": \"copy_oneshot\", \"U1_GBps\": %.1f, \"U2_GBps\": %.1f, \"U4_GBps\": %.1f, \"U8_GBps\": %.1f, "
           "\"cudaMemcpy_d2d_GBps\": %.1f}\n", bytes / (m1 * 1e-3) / 1e9, bytes / (m2 * 1e-3) / 1e9,
           bytes / (m4 * 1e-3) / 1e9, bytes / (m8 * 1e-3) / 1e9, bytes / (mc * 1e-3) / 1e9);
  }
  // fold pattern: N sources of L floats each inside `a`, output in `b`
  for (int N : {8, 16, 32}) {
    const int64_t L = (bytes / 4) / N / 4 * 4;     // floats per source
    Srcs s;
    for (int k = 0; k < N; ++k) s.p[k] = reinterpret_cast<const float *>(a) + k * L;
    const int64_t nv = L / 4;
    const double alg = (double)(N + 1) * L * 4;
    for (int g : {sms * 8, sms * 16, sms * 64}) {
      float m1 = best_ms([&] { k_foldpat<1><<<g, 256>>>(s, N, (float *)b, nv); });
      float m2 = best_ms([&] { k_foldpat<2><<<g, 256>>>(s, N, (float *)b, nv); });
      float m4 = best_ms([&] { k_foldpat<4><<<g, 256>>>(s, N, (float *)b, nv); });
      printf("{\"probe\": \"foldpat\", \"N\": %d, \"grid\": %d, \"U1_GBps\": %.1f, \"U2_GBps\": %.1f, \"U4_GBps\": %.1f}\n",
             N, g, alg / (m1 * 1e-3) / 1e9, alg / (m2 * 1e-3) / 1e9, alg / (m4 * 1e-3) / 1e9);
    }
    {  // one-shot grids (no grid-stride loop), with and without the result write
      const int g1 = (int)((nv + 255) / 256), g2 = (int)((nv / 2 + 255) / 256);
      float m1 = best_ms([&] { k_foldpat<1><<<g1, 256>>>(s, N, (float *)b, nv); });
      float m2 = best_ms([&] { k_foldpat<2><<<g2, 256>>>(s, N, (float *)b, nv); });
      float r1 = best_ms([&] { k_foldpat<1, false><<<g1, 256>>>(s, N, (float *)b, nv); });
      const double rd = (double)N * L * 4;
      printf("{\"probe\": \"foldpat_oneshot\", \"N\": %d, \"grid\": %d, \"U1_GBps\": %.1f, \"U2_GBps\": %.1f, "
             "\"U1_nowrite_read_GBps\": %.1f}\n", N, g1, alg / (m1 * 1e-3) / 1e9, alg / (m2 * 1e-3) / 1e9,
             rd / (r1 * 1e-3) / 1e9);
    }
  }
  {  // bf16, N = 12 (BERT), one-shot grid
    const int N = 12;
    const int64_t L = (bytes / 2) / N / 8 * 8;     // bf16 elements per source
    Srcs s;
    for (int k = 0; k < N; ++k) s.p[k] = reinterpret_cast<const float *>(a + (size_t)k * L * 2);
    const int64_t nv = L / 8;
    const double alg = (double)(N + 1) * L * 2;
    const int g = (int)((nv + 255) / 256);
    float m8 = best_ms([&] { k_foldpat_bf16<8><<<g, 256>>>(s, N, (uint16_t *)b, nv); });
    float m6 = best_ms([&] { k_foldpat_bf16<6><<<g, 256>>>(s, N, (uint16_t *)b, nv); });
    float m12 = best_ms([&] { k_foldpat_bf16<12><<<g, 256>>>(s, N, (uint16_t *)b, nv); });
    float m4 = best_ms([&] { k_foldpat_bf16<4><<<g, 256>>>(s, N, (uint16_t *)b, nv); });
    printf("{\"probe\": \"foldpat_bf16_oneshot\", \"N\": %d, \"grid\": %d, \"B8_GBps\": %.1f, \"B6_GBps\": %.1f, "
           "\"B12_GBps\": %.1f, \"B4_GBps\": %.1f}\n", N, g, alg / (m8 * 1e-3) / 1e9, alg / (m6 * 1e-3) / 1e9,
           alg / (m12 * 1e-3) / 1e9, alg / (m4 * 1e-3) / 1e9);
  }
  CK(cudaGetLastError());
  return 0;
}
