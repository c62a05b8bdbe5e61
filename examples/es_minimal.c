/*
 * es_minimal.c -- the C ABI used directly from C (no Python, no PyTorch):
 * N = 4 ESTs on one GPU, one fp32 bucket of L elements; EST k's gradient is
 * x_k[i] = fl32(v * 0.001f), v = ((i * 2654435761 + 97 k) mod 2001) - 1000
 * (exactly reproducible on any host); ESTs 0..2
 * are stashed (COPY), EST 3 is borrowed, then es_allreduce writes the
 * canonical average.  Writes the L result floats to argv[1] (raw binary) so a
 * test can compare them with the oracle.
 *
 *   gcc -O2 -I include -I /usr/local/cuda/include examples/es_minimal.c -o es_minimal \
 *       -L paper_conf_sc_lixyszrljlllq23_b200 -les -L /usr/local/cuda/lib64 -lcudart -lm
 */
#include <stdio.h>
#include <stdlib.h>

#include <cuda_runtime.h>

#include "es.h"

#define CHECK(call)                                                                    \
  do {                                                                                 \
    es_status s_ = (call);                                                             \
    if (s_ != ES_OK) {                                                                 \
      fprintf(stderr, "%s: %s (%s)\n", #call, es_status_string(s_), es_last_error()); \
      return 1;                                                                        \
    }                                                                                  \
  } while (0)

int main(int argc, char **argv) {
  const int32_t N = 4;
  const uint64_t L = 100003;
  int32_t map[4] = {0, 0, 0, 0};
  es_bucket_desc bucket = {L, ES_F32};
  es_config cfg = {0};
  cfg.N = N;
  cfg.G = 1;
  cfg.rank = 0;
  cfg.est_to_gpu = map;
  cfg.buckets = &bucket;
  cfg.n_buckets = 1;
  cfg.chunk_align = 16;
  cfg.transport = ES_TRANSPORT_NONE;
  cfg.sched = ES_SCHED_AUTO;

  size_t ws_bytes = 0;
  CHECK(es_workspace_bytes(&cfg, &ws_bytes));
  void *ws = NULL, *grads[4], *out = NULL;
  if (cudaMalloc(&ws, ws_bytes) != cudaSuccess || cudaMalloc(&out, L * 4) != cudaSuccess) return 2;
  float *host = (float *)malloc(L * 4);
  for (int k = 0; k < N; ++k) {
    for (uint64_t i = 0; i < L; ++i) {
      const int32_t v = (int32_t)(((uint64_t)i * 2654435761ull + 97ull * (uint64_t)k) % 2001ull) - 1000;
      host[i] = (float)v * 0.001f;
    }
    if (cudaMalloc(&grads[k], L * 4) != cudaSuccess) return 2;
    cudaMemcpy(grads[k], host, L * 4, cudaMemcpyHostToDevice);
  }
  es_handle h = NULL;
  CHECK(es_init(&cfg, ws, ws_bytes, &h));
  for (int k = 0; k < N; ++k)
    CHECK(es_stash_grad(h, k, 0, grads[k], ES_F32, k == N - 1 ? ES_STASH_BORROW : ES_STASH_COPY, NULL));
  CHECK(es_allreduce(h, 0, out, NULL));
  CHECK(es_sync(h));
  cudaMemcpy(host, out, L * 4, cudaMemcpyDeviceToHost);
  CHECK(es_destroy(h));
  if (argc > 1) {
    FILE *f = fopen(argv[1], "wb");
    if (!f || fwrite(host, 4, L, f) != L) return 3;
    fclose(f);
  }
  printf("es_minimal ok: out[1] = %.9g\n", host[1]);
  free(host);
  return 0;
}
