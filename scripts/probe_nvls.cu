// probe_nvls.cu -- NVLink/NVSwitch write rate measured from ONE GPU (not product code).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/probe_nvls scripts/probe_nvls.cu -lcuda
//
// The all-gather of a6 is a pure copy of every rank's result shard to every other
// rank; on NVSwitch it can be one `multimem.st` per element to a multicast address, replicated by
// the switch.  This box shows a single B200, but the GPU reports multicast support
// (CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED) and its 18 NVLinks are up, so a one-member multicast
// object can be built: stores to its multicast mapping leave the GPU over NVLink, are replicated
// by the switch (to the one member) and come back.  The probe times
//   (1) plain 128-bit stores of a source buffer into the unicast mapping (HBM copy),
//   (2) the same stores through the multicast mapping (`multimem.st.global.v4.f32`),
// checks the destination bits, and prints one JSON line per variant.  (2) is an upper bound on
// the per-GPU egress a multimem gather could use on this fabric; it is not a multi-GPU number.
// Result on this pool (profiles/r01_probe_nvls.jsonl): cuMulticastCreate is refused
// (CUDA_ERROR_INVALID_VALUE for every numDevices / handle-type combination) although the attribute
// says multicast is supported -- a one-GPU NVSwitch partition; kept for a multi-GPU box.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstring>
#include <vector>

#define CU(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { const char *s; cuGetErrorString(r, &s); \
  printf("{\"probe\": \"nvls\", \"error\": \"%s: %s\"}\n", #x, s); return 1; } } while (0)
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  printf("{\"probe\": \"nvls\", \"error\": \"%s: %s\"}\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__global__ void __launch_bounds__(256) k_st(const int4 *__restrict__ src, int4 *dst, int64_t nvec) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvec; i += (int64_t)gridDim.x * blockDim.x) {
    int4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(src + i));
    dst[i] = v;
  }
}

__global__ void __launch_bounds__(256) k_mcst(const int4 *__restrict__ src, int4 *mc, int64_t nvec) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvec; i += (int64_t)gridDim.x * blockDim.x) {
    int4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(src + i));
    asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};"
                 :: "l"(mc + i), "f"(__int_as_float(v.x)), "f"(__int_as_float(v.y)), "f"(__int_as_float(v.z)),
                    "f"(__int_as_float(v.w)) : "memory");
  }
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
  CK(cudaSetDevice(0));
  CK(cudaFree(0));
  CUdevice dev;
  CU(cuDeviceGet(&dev, 0));
  int mc_ok = 0, sms = 0;
  CU(cuDeviceGetAttribute(&mc_ok, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
  CU(cuDeviceGetAttribute(&sms, CU_DEVICE_ATTRIBUTE_MULTIPROCESSOR_COUNT, dev));
  printf("{\"probe\": \"nvls\", \"multicast_supported\": %d}\n", mc_ok);
  if (!mc_ok) return 0;

  const size_t want = 1ull << 30;                 // 1 GiB destination
  CUmulticastObjectProp mp;
  memset(&mp, 0, sizeof(mp));
  mp.numDevices = 1;
  mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  mp.size = want;
  size_t gran = 0;
  CU(cuMulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED));
  const size_t size = (want + gran - 1) / gran * gran;
  mp.size = size;
  CUmemGenericAllocationHandle mc, mem;
  {
    // which (numDevices, handle type) combinations does this driver accept for a one-GPU box?
    const struct { unsigned nd; CUmemAllocationHandleType ht; const char *name; } tries[] = {
        {1, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, "1/posix_fd"}, {1, CU_MEM_HANDLE_TYPE_FABRIC, "1/fabric"},
        {1, (CUmemAllocationHandleType)0, "1/none"}, {2, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, "2/posix_fd"}};
    for (auto &t : tries) {
      CUmulticastObjectProp q = mp;
      q.numDevices = t.nd;
      q.handleTypes = t.ht;
      CUmemGenericAllocationHandle x;
      size_t gq = 0;
      CUresult rg = cuMulticastGetGranularity(&gq, &q, CU_MULTICAST_GRANULARITY_RECOMMENDED);
      CUresult r = cuMulticastCreate(&x, &q);
      const char *es = "";
      cuGetErrorString(r, &es);
      printf("{\"probe\": \"nvls\", \"create\": \"%s\", \"granularity_rc\": %d, \"gran\": %zu, \"rc\": %d, \"msg\": \"%s\"}\n",
             t.name, (int)rg, gq, (int)r, es);
      if (r == CUDA_SUCCESS) cuMemRelease(x);
    }
  }
  CU(cuMulticastCreate(&mc, &mp));
  CU(cuMulticastAddDevice(mc, dev));

  CUmemAllocationProp ap;
  memset(&ap, 0, sizeof(ap));
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = 0;
  ap.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  size_t mgran = 0;
  CU(cuMemGetAllocationGranularity(&mgran, &ap, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
  CU(cuMemCreate(&mem, size, &ap, 0));
  CU(cuMulticastBindMem(mc, 0, mem, 0, size, 0));

  CUmemAccessDesc acc;
  memset(&acc, 0, sizeof(acc));
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = 0;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CUdeviceptr uc = 0, mcp = 0;
  CU(cuMemAddressReserve(&uc, size, gran, 0, 0));
  CU(cuMemMap(uc, size, 0, mem, 0));
  CU(cuMemSetAccess(uc, size, &acc, 1));
  CU(cuMemAddressReserve(&mcp, size, gran, 0, 0));
  CU(cuMemMap(mcp, size, 0, mc, 0));
  CU(cuMemSetAccess(mcp, size, &acc, 1));

  const int64_t nvec = (int64_t)(want / 16);
  int4 *src = nullptr;
  CK(cudaMalloc(&src, want));
  std::vector<uint32_t> h(want / 4);
  for (size_t i = 0; i < h.size(); ++i) h[i] = (uint32_t)(i * 2654435761u) & 0x3f7fffffu;  // finite floats
  CK(cudaMemcpy(src, h.data(), want, cudaMemcpyHostToDevice));

  for (int g : {sms * 4, sms * 8, sms * 16, sms * 32}) {
    CK(cudaMemset((void *)uc, 0, want));
    float ms_uc = best_ms([&] { k_st<<<g, 256>>>(src, (int4 *)uc, nvec); });
    CK(cudaGetLastError());
    CK(cudaMemset((void *)uc, 0, want));
    float ms_mc = best_ms([&] { k_mcst<<<g, 256>>>(src, (int4 *)mcp, nvec); });
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    std::vector<uint32_t> back(want / 4);
    CK(cudaMemcpy(back.data(), (void *)uc, want, cudaMemcpyDeviceToHost));
    const bool ok = memcmp(back.data(), h.data(), want) == 0;
    printf("{\"probe\": \"nvls\", \"grid\": %d, \"bytes\": %zu, \"unicast_copy_GBps_rd_plus_wr\": %.1f, "
           "\"multimem_st_GBps_written\": %.1f, \"multimem_bits_ok\": %s}\n",
           g, want, 2.0 * want / (ms_uc * 1e-3) / 1e9, want / (ms_mc * 1e-3) / 1e9, ok ? "true" : "false");
  }
  return 0;
}
