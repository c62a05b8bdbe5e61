// api_peer_context.cpp -- C ABI: peer-memory mapping (ES_SCHED_PEER), zero-copy
// slots, EST context export / import (elastic resume), per-EST dropout.
#include <unistd.h>

#include <chrono>
#include <cstdlib>
#include <random>

#include "handle.h"

extern "C" {

// ---- peer memory ---------------------------------------------------------------------

namespace {

struct PeerBlob {
  char magic[8];            // "ESPEER02"
  int32_t rank, pid;
  uint64_t nonce;           // random per process: pid alone is ambiguous across PID namespaces
  uint64_t plan_hash;       // everything that shapes the peer protocol (must match on every rank)
  uint64_t raw;             // workspace address in the owner's process
  uint64_t offset;          // workspace - allocation base
  uint64_t ws_bytes;
  int32_t ipc_ok, pad;
  cudaIpcMemHandle_t handle;
};
static_assert(sizeof(PeerBlob) <= ES_PEER_BLOB_BYTES, "peer blob too large");

// Base of the allocation that contains p (driver cuMemGetAddressRange,
// resolved through the runtime so libes has no link-time libcuda dependency).
bool allocation_base(void *p, void **base) {
  typedef int (*Fn)(unsigned long long *, size_t *, unsigned long long);
  static Fn fn = nullptr;
  if (!fn) {
    void *sym = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &sym, cudaEnableDefault, &q) != cudaSuccess || !sym) {
      cudaGetLastError();
      return false;
    }
    fn = reinterpret_cast<Fn>(sym);
  }
  unsigned long long b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, (unsigned long long)(uintptr_t)p) != 0) return false;
  *base = reinterpret_cast<void *>((uintptr_t)b);
  return true;
}

uint64_t fnv1a(uint64_t h, const void *p, size_t n) {
  const unsigned char *c = reinterpret_cast<const unsigned char *>(p);
  for (size_t i = 0; i < n; ++i) h = (h ^ c[i]) * 1099511628211ull;
  return h;
}

// One random value per process (ranks in different containers may share a pid).
uint64_t process_nonce() {
  static const uint64_t n = [] {
    std::random_device rd;
    uint64_t x = ((uint64_t)rd() << 32) ^ rd();
    x ^= (uint64_t)std::chrono::steady_clock::now().time_since_epoch().count();
    x ^= (uint64_t)getpid() * 0x9E3779B97F4A7C15ull;
    return x | 1;
  }();
  return n;
}

// Hash of every input that shapes the peer protocol: the layout, N, G, A, the
// mapping, each bucket's schedule, the compat bits and the options (the
// executor's phases, barrier count and gather sources depend on them).  Ranks
// whose plans differ here would wait on barriers the others never reach or
// gather data never pushed.
uint64_t peer_plan_hash(const es::Plan &p) {
  uint64_t h = 1469598103934665603ull;
  h = fnv1a(h, &p.N, sizeof p.N);
  h = fnv1a(h, &p.G, sizeof p.G);
  h = fnv1a(h, &p.A, sizeof p.A);
  h = fnv1a(h, p.est_to_gpu.data(), p.est_to_gpu.size() * sizeof(int32_t));
  for (const es::BucketPlan &b : p.bp) {
    h = fnv1a(h, &b.L, sizeof b.L);
    const int32_t d = (int32_t)b.dtype;
    h = fnv1a(h, &d, sizeof d);
    h = fnv1a(h, &b.sched, sizeof b.sched);
  }
  h = fnv1a(h, &p.compat, sizeof p.compat);
  h = fnv1a(h, &p.options, sizeof p.options);
  return h;
}

}  // namespace

es_status es_peer_blob(es_handle h, void *blob, size_t bytes) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  if (!blob || bytes < ES_PEER_BLOB_BYTES) return set_err(ES_EINVAL, "blob must hold ES_PEER_BLOB_BYTES");
  PeerBlob b;
  std::memset(&b, 0, sizeof b);
  std::memcpy(b.magic, "ESPEER02", 8);
  b.rank = h->plan.rank;
  b.pid = (int32_t)getpid();
  b.nonce = process_nonce();
  b.plan_hash = peer_plan_hash(h->plan);
  b.raw = (uint64_t)(uintptr_t)h->ws;
  b.ws_bytes = h->ws_bytes;
  void *base = nullptr;
  if (allocation_base(h->ws, &base) && cudaIpcGetMemHandle(&b.handle, base) == cudaSuccess) {
    b.ipc_ok = 1;
    b.offset = (uint64_t)((uintptr_t)h->ws - (uintptr_t)base);
  } else {
    cudaGetLastError();
  }
  std::memset(blob, 0, ES_PEER_BLOB_BYTES);
  std::memcpy(blob, &b, sizeof b);
  return ES_OK;
}

es_status es_peer_open(es_handle h, const void *blobs, size_t bytes) {
  ES_NVTX();
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (!blobs || bytes < (size_t)p.G * ES_PEER_BLOB_BYTES) return set_err(ES_EINVAL, "need G blobs");
  if (h->peer_open) return set_err(ES_ESTATE, "peers already open");
  // Peer schedules spin in device barriers: load every kernel now, not on
  // first use (a lazy load waits behind a spinning same-device barrier).
  if (cudaError_t e = es::preload_kernels(); e != cudaSuccess)
    return set_err(ES_ECUDA, std::string("loading the kernels failed: ") + cudaGetErrorString(e));
  std::vector<unsigned char *> ws(p.G, nullptr);
  std::vector<void *> mapped;
  const int32_t me = (int32_t)getpid();
  const uint64_t my_nonce = process_nonce();
  const uint64_t my_hash = peer_plan_hash(p);
  // Ranks sharing this process (loopback) share one device: their barrier
  // kernels spin concurrently on different streams, which needs one hardware
  // queue per rank -- more ranks than CUDA_DEVICE_MAX_CONNECTIONS (default 8)
  // would serialise a spinning barrier in front of a peer's work.
  int32_t same_process = 0;
  for (int32_t g = 0; g < p.G; ++g) {
    PeerBlob b;
    std::memcpy(&b, reinterpret_cast<const unsigned char *>(blobs) + (size_t)g * ES_PEER_BLOB_BYTES, sizeof b);
    same_process += b.pid == me && b.nonce == my_nonce;
  }
  const char *mc = std::getenv("CUDA_DEVICE_MAX_CONNECTIONS");
  const int32_t max_conn = mc ? std::atoi(mc) : 8;
  if (same_process > 1 && same_process > max_conn)
    return set_err(ES_EUNSUPPORTED, "more same-process peer ranks than CUDA_DEVICE_MAX_CONNECTIONS hardware queues");
  for (int32_t g = 0; g < p.G; ++g) {
    PeerBlob b;
    std::memcpy(&b, reinterpret_cast<const unsigned char *>(blobs) + (size_t)g * ES_PEER_BLOB_BYTES, sizeof b);
    if (std::memcmp(b.magic, "ESPEER02", 8) != 0 || b.rank != g) {
      for (void *m : mapped) cudaIpcCloseMemHandle(m);
      return set_err(ES_EINVAL, "blob g is not rank g's es_peer_blob");
    }
    if (b.plan_hash != my_hash) {
      for (void *m : mapped) cudaIpcCloseMemHandle(m);
      return set_err(ES_EINVAL, "rank " + std::to_string(g) +
                                    "'s plan differs (N, G, A, mapping, layout, schedules, compat or options)");
    }
    int32_t n_g = 0;
    for (int32_t e = 0; e < p.N; ++e) n_g += p.est_to_gpu[e] == g;
    if (b.ws_bytes < p.grad_off + (uint64_t)n_g * p.slot_block) {
      for (void *m : mapped) cudaIpcCloseMemHandle(m);
      return set_err(ES_EINVAL, "peer workspace smaller than this layout");
    }
    if (g == p.rank) {
      ws[g] = h->ws;
    } else if (b.pid == me && b.nonce == my_nonce) {
      ws[g] = reinterpret_cast<unsigned char *>((uintptr_t)b.raw);     // same process (loopback)
    } else {
      if (!b.ipc_ok) {
        for (void *m : mapped) cudaIpcCloseMemHandle(m);
        return set_err(ES_EUNSUPPORTED, "peer workspace is not IPC-exportable");
      }
      void *ptr = nullptr;
      if (cudaIpcOpenMemHandle(&ptr, b.handle, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        for (void *m : mapped) cudaIpcCloseMemHandle(m);
        return set_err(ES_ECUDA, "cudaIpcOpenMemHandle failed");
      }
      mapped.push_back(ptr);
      ws[g] = reinterpret_cast<unsigned char *>(ptr) + b.offset;
    }
  }
  h->peer_ws = ws;
  h->ipc_mapped = mapped;
  h->peer_open = true;
  h->peer_share = std::max<int32_t>(1, same_process);
  return ES_OK;
}

// ---- zero-copy slots and elastic resume ------------------------------------------

namespace {

struct CtxHeader {
  char magic[8];           // "ESCTX001"
  uint32_t version;
  int32_t N;
  uint32_t A;
  int32_t n_buckets;
  int32_t n_state;
  int32_t est;
  uint64_t layout_hash;
  uint64_t payload_bytes;
};

uint64_t fnv(uint64_t h, const void *p, size_t n) {
  const unsigned char *c = reinterpret_cast<const unsigned char *>(p);
  for (size_t i = 0; i < n; ++i) h = (h ^ c[i]) * 1099511628211ull;
  return h;
}

// Hash of the persisted layout (D1): N, A, every bucket's numel and dtype,
// every context buffer's size.  G and the mapping are deliberately absent.
uint64_t layout_hash(const es::Plan &p) {
  uint64_t h = 1469598103934665603ull;
  h = fnv(h, &p.N, sizeof p.N);
  h = fnv(h, &p.A, sizeof p.A);
  for (const es_bucket_desc &b : p.buckets) {
    h = fnv(h, &b.numel, sizeof b.numel);
    int32_t d = (int32_t)b.dtype;
    h = fnv(h, &d, sizeof d);
  }
  for (uint64_t n : p.state_nbytes) h = fnv(h, &n, sizeof n);
  h = fnv(h, &p.compat, sizeof p.compat);
  return h;
}

size_t context_bytes(const es::Plan &p) {
  size_t n = sizeof(CtxHeader) + ((p.buckets.size() + 7) & ~size_t(7));
  for (const es::BucketPlan &b : p.bp) n += b.L * b.esize;
  for (uint64_t s : p.state_nbytes) n += s;
  return n;
}

}  // namespace

es_status es_slot_ptr(es_handle h, int32_t est, int32_t bucket, void **ptr) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (!ptr) return set_err(ES_EINVAL, "ptr is NULL");
  if (est < 0 || est >= p.N) return set_err(ES_EINVAL, "est out of range");
  if (bucket < 0 || bucket >= h->B) return set_err(ES_EINVAL, "bucket out of range");
  const int32_t li = p.local_index[est];
  if (li < 0) return set_err(ES_ESTATE, "est is not mapped to this rank");
  *ptr = h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[bucket];
  return ES_OK;
}

es_status es_context_bytes(es_handle h, size_t *bytes) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  if (!bytes) return set_err(ES_EINVAL, "bytes is NULL");
  *bytes = context_bytes(h->plan);
  return ES_OK;
}

es_status es_export_context(es_handle h, int32_t est, void *host_dst, size_t bytes, es_stream stream) {
  ES_NVTX();
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (!host_dst) return set_err(ES_EINVAL, "host_dst is NULL");
  if (bytes < context_bytes(p)) return set_err(ES_EINVAL, "buffer smaller than es_context_bytes()");
  if (est < 0 || est >= p.N) return set_err(ES_EINVAL, "est out of range");
  const int32_t li = p.local_index[est];
  if (li < 0) return set_err(ES_ESTATE, "est is not mapped to this rank");
  const int32_t nst = (int32_t)p.state_nbytes.size();
  if (nst > 0 && !h->state_registered) return set_err(ES_ESTATE, "es_register_state has not been called");
  // NEXT-1: a COPY stash of a bucket being folded incrementally keeps only
  // the chunks that wait for the wrap in the slot (the rest went into the
  // fp32 partials), so the slot is not this EST's gradient: refuse.
  for (int32_t b = 0; b < h->B; ++b) {
    const size_t k = (size_t)li * h->B + b;
    if (h->inc_next[b] > 0 && h->stashed[k] && !h->borrowed[k] && h->inc_full[k] == 0)
      return set_err(ES_ESTATE, "bucket is being folded incrementally (es_stash_fold_grads): its slot holds "
                                "only part of the EST's gradient and cannot be exported");
  }
  cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
  unsigned char *o = reinterpret_cast<unsigned char *>(host_dst);
  CtxHeader hd;
  std::memset(&hd, 0, sizeof hd);
  std::memcpy(hd.magic, "ESCTX001", 8);
  hd.version = 1;
  hd.N = p.N;
  hd.A = p.A;
  hd.n_buckets = h->B;
  hd.n_state = nst;
  hd.est = est;
  hd.layout_hash = layout_hash(p);
  hd.payload_bytes = context_bytes(p);
  std::memcpy(o, &hd, sizeof hd);
  unsigned char *mask = o + sizeof hd;
  size_t off = sizeof hd + ((p.buckets.size() + 7) & ~size_t(7));
  std::memset(mask, 0, off - sizeof hd);
  for (int32_t b = 0; b < h->B; ++b) {
    const es::BucketPlan &bp = p.bp[b];
    const size_t k = (size_t)li * h->B + b;
    const size_t nb = bp.L * bp.esize;
    if (h->stashed[k] && nb > 0) {
      mask[b] = 1;
      const void *src = h->borrowed[k] ? h->borrowed[k]
                                       : (const void *)(h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[b]);
      if (h->stash_cap[k] == 0 && cudaStreamWaitEvent(cs, h->stash_ev[k], 0) != cudaSuccess)
        return h->poison(ES_ECUDA, "cudaStreamWaitEvent failed");
      if (cudaMemcpyAsync(o + off, src, nb, cudaMemcpyDeviceToHost, cs) != cudaSuccess)
        return h->poison(ES_ECUDA, "cudaMemcpyAsync D2H of a stashed bucket failed");
    } else {
      mask[b] = h->stashed[k] ? 1 : 0;
      std::memset(o + off, 0, nb);
    }
    off += nb;
  }
  for (int32_t i = 0; i < nst; ++i) {
    const void *src = li == h->cur_local ? h->live_ptr[i]
                                         : (const void *)(h->ws + p.state_area_off + (uint64_t)li * p.state_block +
                                                          p.state_off[i]);
    if (cudaMemcpyAsync(o + off, src, p.state_nbytes[i], cudaMemcpyDeviceToHost, cs) != cudaSuccess)
      return h->poison(ES_ECUDA, "cudaMemcpyAsync D2H of EST state failed");
    off += p.state_nbytes[i];
  }
  if (cudaStreamSynchronize(cs) != cudaSuccess) return h->poison(ES_ECUDA, "cudaStreamSynchronize failed");
  return ES_OK;
}

es_status es_import_context(es_handle h, int32_t est, const void *host_src, size_t bytes, es_stream stream) {
  ES_NVTX();
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (!host_src) return set_err(ES_EINVAL, "host_src is NULL");
  if (bytes < sizeof(CtxHeader)) return set_err(ES_EINVAL, "blob too small");
  CtxHeader hd;
  std::memcpy(&hd, host_src, sizeof hd);
  if (std::memcmp(hd.magic, "ESCTX001", 8) != 0 || hd.version != 1) return set_err(ES_EINVAL, "not an es context blob");
  if (hd.layout_hash != layout_hash(p) || hd.N != p.N || hd.A != p.A || hd.n_buckets != h->B)
    return set_err(ES_ESTATE, "context was exported under a different N / A / bucket layout (D1 mismatch)");
  if (bytes < context_bytes(p) || hd.payload_bytes != context_bytes(p)) return set_err(ES_EINVAL, "blob truncated");
  if (est < 0 || est >= p.N) return set_err(ES_EINVAL, "est out of range");
  if (hd.est != est) return set_err(ES_EINVAL, "blob belongs to another EST");
  const int32_t li = p.local_index[est];
  if (li < 0) return set_err(ES_ESTATE, "est is not mapped to this rank");
  const int32_t nst = (int32_t)p.state_nbytes.size();
  if (nst > 0 && li == h->cur_local && !h->state_registered)
    return set_err(ES_ESTATE, "es_register_state has not been called");
  {
    const unsigned char *m = reinterpret_cast<const unsigned char *>(host_src) + sizeof hd;
    for (int32_t b = 0; b < h->B; ++b)
      if (m[b] && h->inc_next[b] > 0)
        return set_err(ES_ESTATE, "bucket is being folded incrementally this step: an imported contribution "
                                  "would bypass the running partials");
  }
  cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
  const unsigned long long cap = capture_id(cs);
  const unsigned char *in = reinterpret_cast<const unsigned char *>(host_src);
  const unsigned char *mask = in + sizeof hd;
  size_t off = sizeof hd + ((p.buckets.size() + 7) & ~size_t(7));
  for (int32_t b = 0; b < h->B; ++b) {
    const es::BucketPlan &bp = p.bp[b];
    const size_t k = (size_t)li * h->B + b;
    const size_t nb = bp.L * bp.esize;
    if (mask[b]) {
      unsigned char *dst = h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[b];
      if (h->ar_recorded[b] && h->ar_cap[b] == cap && cudaStreamWaitEvent(cs, h->ar_ev[b], 0) != cudaSuccess)
        return h->poison(ES_ECUDA, "cudaStreamWaitEvent failed");
      if (nb > 0 && cudaMemcpyAsync(dst, in + off, nb, cudaMemcpyHostToDevice, cs) != cudaSuccess)
        return h->poison(ES_ECUDA, "cudaMemcpyAsync H2D of a stashed bucket failed");
      h->borrowed[k] = nullptr;
      if (cudaEventRecord(h->stash_ev[k], cs) != cudaSuccess) return h->poison(ES_ECUDA, "cudaEventRecord failed");
      h->stash_cap[k] = cap;
      h->stashed[k] = 1;
    }
    off += nb;
  }
  for (int32_t i = 0; i < nst; ++i) {
    void *dst = li == h->cur_local ? h->live_ptr[i]
                                   : (void *)(h->ws + p.state_area_off + (uint64_t)li * p.state_block + p.state_off[i]);
    if (cudaMemcpyAsync(dst, in + off, p.state_nbytes[i], cudaMemcpyHostToDevice, cs) != cudaSuccess)
      return h->poison(ES_ECUDA, "cudaMemcpyAsync H2D of EST state failed");
    off += p.state_nbytes[i];
  }
  // host_src may be released by the caller on return
  if (cudaStreamSynchronize(cs) != cudaSuccess) return h->poison(ES_ECUDA, "cudaStreamSynchronize failed");
  return ES_OK;
}

// ---- NEXT-4: per-EST dropout ---------------------------------------------------

es_status es_dropout(es_handle h, const void *x, void *y, uint8_t *mask, uint64_t n, es_dtype dtype, float p,
                     int32_t state_idx, es_stream stream) {
  ES_NVTX();
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &pl = h->plan;
  if (dtype != ES_F32 && dtype != ES_BF16) return set_err(ES_EINVAL, "bad dtype");
  if (!(p >= 0.0f && p < 1.0f)) return set_err(ES_EINVAL, "p must be in [0, 1)");
  if (n >= (1ull << 40)) return set_err(ES_EINVAL, "n too large");
  if (n > 0 && (!x || !y)) return set_err(ES_EINVAL, "x / y are NULL");
  if (state_idx < 0 || state_idx >= (int32_t)pl.state_nbytes.size() || pl.state_nbytes[state_idx] != 16)
    return set_err(ES_EINVAL, "state_idx must name a registered 16-byte Philox record");
  if (!h->state_registered) return set_err(ES_ESTATE, "es_register_state has not been called");
  if (h->cur_local < 0) return set_err(ES_ESTATE, "no EST is running (call es_switch_context first)");
  cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
  const float scale = 1.0f / (1.0f - p);
  const uint64_t nbytes = n * (2 * (uint64_t)es::dtype_size(dtype) + (mask ? 1 : 0));
  return h->timed(ES_KERNEL_DROPOUT, nbytes, cs, [&](int *nl) {
    *nl = 1;
    return es::launch_dropout(dtype, x, y, mask, (int64_t)n, p, scale,
                              reinterpret_cast<uint64_t *>(h->live_ptr[state_idx]),
                              reinterpret_cast<unsigned int *>(h->ws + pl.scratch_off), cs);
  });
}


}  // extern "C"
