// es_api.cpp -- the C ABI of libes (include/es.h): argument checking, the
// per-rank handle, stash bookkeeping, and the executor that walks the
// planner's op list (plan.cpp) launching kernels (kernels.cu) and transport
// groups (transport_*.cpp) on the caller's stream.
#include <cuda_runtime.h>

#include <unistd.h>

#include <algorithm>
#include <cstring>
#include <memory>
#include <string>
#include <vector>

#include "../../include/es.h"
#include "kernels.h"
#include "plan.h"
#include "transport.h"

namespace {

thread_local std::string g_err;

es_status set_err(es_status s, const std::string &msg) {
  g_err = msg;
  return s;
}

bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// CUDA-graph support: the id of the capture `s` is part of, 0 when eager.
// Events recorded in one capture (or eagerly) are only waited on from the
// same capture (or eagerly): a graph cannot depend on work outside it, and
// replays of a graph on one stream are ordered anyway.
unsigned long long capture_id(cudaStream_t s) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  unsigned long long id = 0;
  if (cudaStreamGetCaptureInfo(s, &st, &id) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return st == cudaStreamCaptureStatusActive ? id : 0;
}

}  // namespace

struct es_ctx {
  es::Plan plan;
  unsigned char *ws = nullptr;
  size_t ws_bytes = 0;
  std::unique_ptr<es::Transport> tp;
  int device = 0;
  int32_t B = 0, n_local = 0;

  // stash bookkeeping, [local EST index * B + bucket]
  std::vector<uint8_t> stashed;
  std::vector<const void *> borrowed;
  std::vector<cudaEvent_t> stash_ev;
  std::vector<unsigned long long> stash_cap;
  std::vector<cudaEvent_t> ar_ev;       // [B]: last es_allreduce of the bucket
  std::vector<unsigned long long> ar_cap;
  std::vector<uint8_t> ar_recorded;
  cudaEvent_t last_ar = nullptr;        // orders staging / partial reuse across buckets
  unsigned long long last_ar_cap = 0;

  // context state
  bool state_registered = false;
  std::vector<void *> live_ptr;
  uint64_t max_state = 0;
  int32_t cur_local = -1;

  es_status sticky = ES_OK;
  std::string sticky_msg;

  // NEXT-1 incremental fold: next EST expected per bucket (0: none folded yet)
  std::vector<int32_t> inc_next;

  // ES_SCHED_PEER
  std::vector<unsigned char *> peer_ws;   // [G] workspace base of every rank, mapped here
  std::vector<void *> ipc_mapped;         // cudaIpcOpenMemHandle results to close
  bool peer_open = false;
  uint64_t barrier_epoch = 0;

  // instrumentation
  bool prof = false;
  struct Rec {
    int kind;
    cudaEvent_t a, b;
    bool captured;       // recorded by a CUDA-graph node: never recycled
  };
  std::vector<Rec> recs;
  std::vector<cudaEvent_t> pool;
  std::vector<cudaEvent_t> graph_events;
  uint64_t launches[ES_KERNEL_KINDS] = {};
  uint64_t bytes[ES_KERNEL_KINDS] = {};
  double ms[ES_KERNEL_KINDS] = {};
  int blocks_ov = 0, threads_ov = 0;

  ~es_ctx() {
    for (auto e : stash_ev) if (e) cudaEventDestroy(e);
    for (auto e : ar_ev) if (e) cudaEventDestroy(e);
    for (auto &r : recs) { cudaEventDestroy(r.a); cudaEventDestroy(r.b); }
    for (auto e : pool) cudaEventDestroy(e);
    for (auto e : graph_events) cudaEventDestroy(e);
    for (void *p : ipc_mapped) cudaIpcCloseMemHandle(p);
  }
  cudaEvent_t ev() {
    if (!pool.empty()) {
      cudaEvent_t e = pool.back();
      pool.pop_back();
      return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
  }
  es_status poison(es_status s, const std::string &msg) {
    if (sticky == ES_OK) {
      sticky = s;
      sticky_msg = msg;
    }
    return set_err(s, msg);
  }
  es_status check_sticky() {
    if (sticky != ES_OK) return set_err(sticky, "handle poisoned by an earlier error: " + sticky_msg);
    return ES_OK;
  }
  // Runs `launch(int* n_launches)` bracketed by timing events when profiling is on.
  template <typename F>
  es_status timed(int kind, uint64_t nbytes, cudaStream_t s, F launch) {
    cudaEvent_t a = nullptr, b = nullptr;
    // Inside a graph capture the timing events become event-record nodes.
    const bool cap = capture_id(s) != 0;
    const unsigned int flags = cap ? cudaEventRecordExternal : cudaEventRecordDefault;
    if (prof) {
      a = ev();
      b = ev();
      cudaEventRecordWithFlags(a, s, flags);
    }
    int n = 0;
    cudaError_t e = launch(&n);
    if (e != cudaSuccess) return poison(ES_ECUDA, std::string("kernel launch: ") + cudaGetErrorString(e));
    if (prof) {
      cudaEventRecordWithFlags(b, s, flags);
      recs.push_back({kind, a, b, cap});
    }
    launches[kind] += n;
    bytes[kind] += nbytes;
    return ES_OK;
  }
};

namespace {

es_status check_handle(es_handle h) {
  if (!h) return set_err(ES_EINVAL, "handle is NULL");
  return h->check_sticky();
}

}  // namespace

extern "C" {

int32_t es_abi_version(void) { return ES_ABI_VERSION; }

const char *es_status_string(es_status s) {
  switch (s) {
    case ES_OK: return "ES_OK";
    case ES_EINVAL: return "ES_EINVAL: invalid argument";
    case ES_ESTATE: return "ES_ESTATE: protocol violation";
    case ES_ENOMEM: return "ES_ENOMEM: workspace too small";
    case ES_ECUDA: return "ES_ECUDA: CUDA error";
    case ES_ENCCL: return "ES_ENCCL: NCCL error";
    case ES_EUNSUPPORTED: return "ES_EUNSUPPORTED: unsupported";
  }
  return "unknown es_status";
}

const char *es_last_error(void) { return g_err.c_str(); }

uint64_t es_chunk_elems(uint64_t L, int32_t N, uint32_t A) { return es::chunk_elems(L, N, A ? A : 16); }

es_status es_workspace_bytes(const es_config *cfg, size_t *bytes) {
  if (!bytes) return set_err(ES_EINVAL, "bytes is NULL");
  es::Plan p;
  std::string err;
  es_status s = es::build_plan(cfg, &p, &err, false);
  if (s != ES_OK) return set_err(s, err);
  *bytes = p.total;
  return ES_OK;
}

es_status es_plan_ops(const es_config *cfg, int32_t bucket, int64_t *ops, size_t cap_ops, size_t *n_ops,
                      int32_t *sched_out) {
  if (!n_ops) return set_err(ES_EINVAL, "n_ops is NULL");
  es::Plan p;
  std::string err;
  es_status s = es::build_plan(cfg, &p, &err, false);
  if (s != ES_OK) return set_err(s, err);
  if (bucket < 0 || bucket >= (int32_t)p.bp.size()) return set_err(ES_EINVAL, "bucket out of range");
  const es::BucketPlan &b = p.bp[bucket];
  *n_ops = b.ops.size();
  if (sched_out) *sched_out = b.sched;
  if (ops)
    for (size_t i = 0; i < b.ops.size() && i < cap_ops; ++i)
      std::memcpy(ops + i * ES_OP_FIELDS, b.ops[i].f, sizeof(int64_t) * ES_OP_FIELDS);
  return ES_OK;
}

es_status es_init(const es_config *cfg, void *workspace, size_t workspace_bytes, es_handle *out) {
  if (!out) return set_err(ES_EINVAL, "out is NULL");
  *out = nullptr;
  std::unique_ptr<es_ctx> h(new es_ctx());
  std::string err;
  es_status s = es::build_plan(cfg, &h->plan, &err);
  if (s != ES_OK) return set_err(s, err);
  if (!workspace || (reinterpret_cast<uintptr_t>(workspace) & 255u))
    return set_err(ES_EINVAL, "workspace must be a non-NULL 256-byte aligned device pointer");
  if (workspace_bytes < h->plan.total)
    return set_err(ES_ENOMEM, "workspace smaller than es_workspace_bytes()");
  cudaPointerAttributes attr;
  if (cudaPointerGetAttributes(&attr, workspace) != cudaSuccess || attr.type != cudaMemoryTypeDevice) {
    cudaGetLastError();
    return set_err(ES_EINVAL, "workspace is not device memory");
  }
  if (cudaGetDevice(&h->device) != cudaSuccess) return set_err(ES_ECUDA, "cudaGetDevice failed");
  h->ws = reinterpret_cast<unsigned char *>(workspace);
  h->ws_bytes = workspace_bytes;
  h->B = (int32_t)h->plan.bp.size();
  h->n_local = (int32_t)h->plan.local_ests.size();
  const size_t nslot = (size_t)h->B * h->n_local;
  h->stashed.assign(nslot, 0);
  h->borrowed.assign(nslot, nullptr);
  h->stash_ev.assign(nslot, nullptr);
  h->stash_cap.assign(nslot, 0);
  h->ar_ev.assign(h->B, nullptr);
  h->ar_cap.assign(h->B, 0);
  h->ar_recorded.assign(h->B, 0);
  h->inc_next.assign(h->B, 0);
  for (auto &e : h->stash_ev)
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
      return set_err(ES_ECUDA, "cudaEventCreate failed");
  for (auto &e : h->ar_ev)
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
      return set_err(ES_ECUDA, "cudaEventCreate failed");
  for (uint64_t n : h->plan.state_nbytes) h->max_state = std::max<uint64_t>(h->max_state, n);
  if (cudaMemset(h->ws + h->plan.scratch_off, 0, 256) != cudaSuccess) return set_err(ES_ECUDA, "cudaMemset failed");
  if (h->plan.peer && cudaMemset(h->ws + h->plan.flags_off, 0, 64 * 8) != cudaSuccess)
    return set_err(ES_ECUDA, "cudaMemset of the peer flags failed");
  if (h->plan.G > 1 && h->plan.transport != ES_TRANSPORT_NONE) {
    es::Transport *t = h->plan.transport == ES_TRANSPORT_NCCL
                           ? es::make_nccl_transport(h->plan.comm, h->plan.G, h->plan.rank, &err)
                           : es::make_loopback_transport(h->plan.comm, h->plan.G, h->plan.rank, &err);
    if (!t) return set_err(h->plan.transport == ES_TRANSPORT_NCCL ? ES_ENCCL : ES_EINVAL, err);
    h->tp.reset(t);
  }
  *out = h.release();
  return ES_OK;
}

es_status es_destroy(es_handle h) {
  if (!h) return set_err(ES_EINVAL, "handle is NULL");
  delete h;
  return ES_OK;
}

es_status es_sync(es_handle h) {
  if (!h) return set_err(ES_EINVAL, "handle is NULL");
  es_status s = h->check_sticky();
  if (s != ES_OK) return s;
  cudaError_t e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaGetLastError();
  if (e != cudaSuccess) return h->poison(ES_ECUDA, std::string("asynchronous CUDA error: ") + cudaGetErrorString(e));
  return ES_OK;
}

// ---- context state ----------------------------------------------------------

es_status es_register_state(es_handle h, int32_t n, void *const *live) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (n != (int32_t)p.state_nbytes.size()) return set_err(ES_EINVAL, "n must equal cfg.n_state");
  if (n > 0 && !live) return set_err(ES_EINVAL, "live_dev_ptrs is NULL");
  std::vector<es::SwapEntry> tab(n);
  for (int32_t i = 0; i < n; ++i) {
    if (!live[i] || !aligned16(live[i])) return set_err(ES_EINVAL, "live state pointers must be 16-byte aligned");
    tab[i].live = reinterpret_cast<unsigned char *>(live[i]);
    tab[i].slot0 = h->ws + p.state_area_off + p.state_off[i];
    tab[i].stride = p.state_block;
    tab[i].nbytes = p.state_nbytes[i];
  }
  if (n > 0 && cudaMemcpy(h->ws + p.table_off, tab.data(), sizeof(es::SwapEntry) * n, cudaMemcpyHostToDevice) !=
                   cudaSuccess)
    return h->poison(ES_ECUDA, "cudaMemcpy of the swap table failed");
  h->live_ptr.assign(live, live + n);
  h->state_registered = true;
  return ES_OK;
}

static es_status state_slot(es_handle h, int32_t est, int32_t idx, unsigned char **ptr, uint64_t *nbytes) {
  const es::Plan &p = h->plan;
  if (est < 0 || est >= p.N) return set_err(ES_EINVAL, "est out of range");
  if (idx < 0 || idx >= (int32_t)p.state_nbytes.size()) return set_err(ES_EINVAL, "state idx out of range");
  int32_t li = p.local_index[est];
  if (li < 0) return set_err(ES_ESTATE, "est is not mapped to this rank");
  *ptr = h->ws + p.state_area_off + (uint64_t)li * p.state_block + p.state_off[idx];
  *nbytes = p.state_nbytes[idx];
  return ES_OK;
}

es_status es_init_state(es_handle h, int32_t est, int32_t idx, const void *host_src) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  if (!host_src) return set_err(ES_EINVAL, "host_src is NULL");
  unsigned char *d;
  uint64_t nb;
  if ((s = state_slot(h, est, idx, &d, &nb)) != ES_OK) return s;
  if (cudaMemcpy(d, host_src, nb, cudaMemcpyHostToDevice) != cudaSuccess)
    return h->poison(ES_ECUDA, "cudaMemcpy H2D of EST state failed");
  return ES_OK;
}

es_status es_read_state(es_handle h, int32_t est, int32_t idx, void *host_dst) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  if (!host_dst) return set_err(ES_EINVAL, "host_dst is NULL");
  unsigned char *d;
  uint64_t nb;
  if ((s = state_slot(h, est, idx, &d, &nb)) != ES_OK) return s;
  if (cudaMemcpy(host_dst, d, nb, cudaMemcpyDeviceToHost) != cudaSuccess)
    return h->poison(ES_ECUDA, "cudaMemcpy D2H of EST state failed");
  return ES_OK;
}

es_status es_switch_context(es_handle h, int32_t est, es_stream stream) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (est < 0 || est >= p.N) return set_err(ES_EINVAL, "est out of range");
  int32_t li = p.local_index[est];
  if (li < 0) return set_err(ES_ESTATE, "est is not mapped to this rank");
  const int32_t n = (int32_t)p.state_nbytes.size();
  if (n > 0 && !h->state_registered) return set_err(ES_ESTATE, "es_register_state has not been called");
  if (li == h->cur_local) return ES_OK;
  if (n > 0) {
    uint64_t tot = 0;
    for (uint64_t b : p.state_nbytes) tot += b;
    cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
    const int32_t cur = h->cur_local;
    const auto *tab = reinterpret_cast<const es::SwapEntry *>(h->ws + p.table_off);
    s = h->timed(ES_KERNEL_SWAP, (cur >= 0 ? 4 : 2) * tot, cs,
                 [&](int *nl) {
                   *nl = 1;
                   return es::launch_swap(tab, n, h->max_state, cur, li, cs);
                 });
    if (s != ES_OK) return s;
  }
  h->cur_local = li;
  return ES_OK;
}

// ---- stash ----------------------------------------------------------------------

namespace {

// Stash of `n` buckets of local EST `est`, optionally fused with a context
// switch to local EST `next_est` (-1: no switch) in the same launch.
es_status stash_impl(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                     const es_dtype *gdts, es_stash_mode mode, int32_t next_est, es_stream stream) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (n < 0 || (n > 0 && (!buckets || !grads || !gdts))) return set_err(ES_EINVAL, "bad bucket/grad arrays");
  if (est < 0 || est >= p.N) return set_err(ES_EINVAL, "est out of range");
  if (mode != ES_STASH_COPY && mode != ES_STASH_BORROW && mode != ES_STASH_INPLACE)
    return set_err(ES_EINVAL, "bad stash mode");
  for (int32_t i = 0; i < n; ++i) {
    const int32_t bk = buckets[i];
    if (bk < 0 || bk >= h->B) return set_err(ES_EINVAL, "bucket out of range");
    if (gdts[i] != ES_F32 && gdts[i] != ES_BF16) return set_err(ES_EINVAL, "bad grad dtype");
    const es::BucketPlan &b = p.bp[bk];
    if (b.L > 0 && (!grads[i] || !aligned16(grads[i])))
      return set_err(ES_EINVAL, "grad must be a 16-byte aligned device pointer");
    if (mode != ES_STASH_COPY && gdts[i] != b.dtype)
      return set_err(ES_EINVAL, "BORROW / INPLACE need grad dtype == bucket dtype");
  }
  const int32_t li = p.local_index[est];
  if (li < 0) return set_err(ES_ESTATE, "est is not mapped to this rank");
  for (int32_t i = 0; i < n; ++i)
    if (h->inc_next[buckets[i]] > 0)
      return set_err(ES_ESTATE, "bucket is being folded incrementally this step (es_stash_fold_grads)");
  if (mode == ES_STASH_INPLACE)
    for (int32_t i = 0; i < n; ++i)
      if (p.bp[buckets[i]].L > 0 &&
          grads[i] != h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[buckets[i]])
        return set_err(ES_EINVAL, "INPLACE needs grad == es_slot_ptr(est, bucket)");
  // optional fused context switch
  es::SwapArgs swap;
  int32_t next_li = h->cur_local;
  if (next_est >= 0) {
    if (next_est >= p.N) return set_err(ES_EINVAL, "next est out of range");
    next_li = p.local_index[next_est];
    if (next_li < 0) return set_err(ES_ESTATE, "next est is not mapped to this rank");
    const int32_t nst = (int32_t)p.state_nbytes.size();
    if (nst > 0 && !h->state_registered) return set_err(ES_ESTATE, "es_register_state has not been called");
    if (nst > 0 && next_li != h->cur_local) {
      swap.tab = reinterpret_cast<const es::SwapEntry *>(h->ws + p.table_off);
      swap.n = nst;
      swap.max_nbytes = h->max_state;
      swap.cur = h->cur_local;
      swap.next = next_li;
    }
  }
  uint64_t swap_bytes = 0;
  for (uint64_t b : p.state_nbytes) swap_bytes += b;
  swap_bytes *= swap.cur >= 0 ? 4 : 2;
  cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
  const unsigned long long cap = capture_id(cs);
  bool swapped = swap.n == 0;
  if (mode == ES_STASH_COPY) {
    // A slot may be overwritten only after the previous aggregation of its bucket read it.
    for (int32_t i = 0; i < n; ++i) {
      const int32_t bk = buckets[i];
      if (h->ar_recorded[bk] && h->ar_cap[bk] == cap && cudaStreamWaitEvent(cs, h->ar_ev[bk], 0) != cudaSuccess)
        return h->poison(ES_ECUDA, "cudaStreamWaitEvent failed");
    }
    // One multi-segment launch per (grad dtype, bucket dtype) pair present.
    for (int sd = 0; sd < 2; ++sd)
      for (int dd = 0; dd < 2; ++dd) {
        std::vector<es::StashSegDesc> segs;
        uint64_t nbytes = 0;
        for (int32_t i = 0; i < n; ++i) {
          const int32_t bk = buckets[i];
          const es::BucketPlan &b = p.bp[bk];
          if ((int)gdts[i] != sd || (int)b.dtype != dd || b.L == 0) continue;
          segs.push_back({grads[i], h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[bk], (int64_t)b.L});
          nbytes += b.L * (es::dtype_size(gdts[i]) + b.esize);
        }
        if (segs.empty()) continue;
        const es::SwapArgs *sw = swapped ? nullptr : &swap;
        s = h->timed(ES_KERNEL_STASH, nbytes + (sw ? swap_bytes : 0), cs, [&](int *nl) {
          return es::launch_stash_multi((es_dtype)sd, (es_dtype)dd, segs.data(), (int)segs.size(), cs, h->blocks_ov,
                                        h->threads_ov, nl, sw);
        });
        if (s != ES_OK) return s;
        swapped = true;
      }
  }
  if (!swapped) {   // BORROW (or nothing to copy): the switch runs alone
    s = h->timed(ES_KERNEL_SWAP, swap_bytes, cs, [&](int *nl) {
      *nl = 1;
      return es::launch_swap(swap.tab, swap.n, swap.max_nbytes, swap.cur, swap.next, cs);
    });
    if (s != ES_OK) return s;
  }
  h->cur_local = next_li;
  for (int32_t i = 0; i < n; ++i) {
    const size_t k = (size_t)li * h->B + buckets[i];
    h->borrowed[k] = mode == ES_STASH_BORROW ? grads[i] : nullptr;   // INPLACE: the slot itself
    if (cudaEventRecord(h->stash_ev[k], cs) != cudaSuccess) return h->poison(ES_ECUDA, "cudaEventRecord failed");
    h->stash_cap[k] = cap;
    h->stashed[k] = 1;
  }
  return ES_OK;
}

}  // namespace

es_status es_stash_grads(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                         const es_dtype *gdts, es_stash_mode mode, es_stream stream) {
  return stash_impl(h, est, n, buckets, grads, gdts, mode, -1, stream);
}

es_status es_stash_fold_grads(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                              const es_dtype *gdts, es_stash_mode mode, es_stream stream) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (!(p.options & ES_OPT_INCREMENTAL) || p.G != 1)
    return set_err(ES_EUNSUPPORTED, "es_stash_fold_grads needs G == 1 and ES_OPT_INCREMENTAL");
  if (n < 0 || (n > 0 && (!buckets || !grads || !gdts))) return set_err(ES_EINVAL, "bad bucket/grad arrays");
  if (est < 0 || est >= p.N) return set_err(ES_EINVAL, "est out of range");
  if (mode != ES_STASH_COPY && mode != ES_STASH_BORROW) return set_err(ES_EINVAL, "mode must be COPY or BORROW");
  for (int32_t i = 0; i < n; ++i) {
    const int32_t bk = buckets[i];
    if (bk < 0 || bk >= h->B) return set_err(ES_EINVAL, "bucket out of range");
    const es::BucketPlan &b = p.bp[bk];
    if (gdts[i] != b.dtype) return set_err(ES_EINVAL, "incremental fold needs grad dtype == bucket dtype");
    if (b.L > 0 && (!grads[i] || !aligned16(grads[i])))
      return set_err(ES_EINVAL, "grad must be a 16-byte aligned device pointer");
    for (int32_t j = 0; j < i; ++j)
      if (buckets[j] == bk) return set_err(ES_EINVAL, "bucket listed twice");
    if (h->inc_next[bk] != est)
      return set_err(ES_ESTATE, "incremental fold expects the ESTs of a bucket in order 0, 1, ..., N-1");
    if (est == 0)
      for (int32_t li = 0; li < h->n_local; ++li)
        if (h->stashed[(size_t)li * h->B + bk])
          return set_err(ES_ESTATE, "bucket already stashed this step with es_stash_grad(s)");
  }
  const int32_t li = p.local_index[est];
  cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
  const unsigned long long cap = capture_id(cs);
  for (int32_t i = 0; i < n; ++i) {
    const int32_t bk = buckets[i];
    if (h->ar_recorded[bk] && h->ar_cap[bk] == cap && cudaStreamWaitEvent(cs, h->ar_ev[bk], 0) != cudaSuccess)
      return h->poison(ES_ECUDA, "cudaStreamWaitEvent failed");
  }
  const float r = 1.0f / (float)p.N;
  for (int dd = 0; dd < 2; ++dd) {
    // (i) fold x_est into the partials of chunks c < est (R2: est follows c+1..est-1)
    std::vector<es::FoldSegDesc> segs;
    std::vector<std::vector<const void *>> srcs;
    uint64_t fbytes = 0;
    // (ii) stash chunks >= est (they wait for the wrap)
    std::vector<es::StashSegDesc> st;
    uint64_t sbytes = 0;
    for (int32_t i = 0; i < n; ++i) {
      const int32_t bk = buckets[i];
      const es::BucketPlan &b = p.bp[bk];
      if ((int)b.dtype != dd || b.L == 0) continue;
      const unsigned char *x = reinterpret_cast<const unsigned char *>(grads[i]);
      float *part = reinterpret_cast<float *>(h->ws + p.inc_off + p.inc_bucket_off[bk]);
      const int64_t L = (int64_t)b.L, C = (int64_t)b.C;
      const int64_t cont_hi = std::min<int64_t>(L, (int64_t)std::max(est - 1, 0) * C);   // chunks < est-1
      const int64_t inc_hi = std::min<int64_t>(L, (int64_t)est * C);                     // chunks < est
      auto add = [&](int64_t lo, int64_t hi, bool cont) {
        if (hi <= lo) return;
        es::FoldSegDesc d;
        d.lo = lo;
        d.n = hi - lo;
        d.C = (uint32_t)b.C;
        d.rot = false;
        d.m = 1;
        d.part_in = cont ? part + lo : nullptr;
        d.out_partial = true;
        d.out = part + lo;
        segs.push_back(d);
        srcs.push_back({x + (uint64_t)lo * b.esize});
        fbytes += (uint64_t)(hi - lo) * (b.esize + (cont ? 8 : 4));
      };
      add(0, cont_hi, true);           // partial continues
      add(cont_hi, inc_hi, false);     // chunk est-1: est is its first EST (c+1)
      if (mode == ES_STASH_COPY && inc_hi < L) {
        unsigned char *slot = h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[bk];
        st.push_back({x + (uint64_t)inc_hi * b.esize, slot + (uint64_t)inc_hi * b.esize, L - inc_hi});
        sbytes += 2 * (uint64_t)(L - inc_hi) * b.esize;
      }
    }
    if (!segs.empty()) {
      for (size_t j = 0; j < segs.size(); ++j) segs[j].src = srcs[j].data();
      s = h->timed(ES_KERNEL_FOLD, fbytes, cs, [&](int *nl) {
        return es::launch_fold_multi((es_dtype)dd, p.N, r, p.compat, segs.data(), (int)segs.size(), cs, h->blocks_ov,
                                     h->threads_ov, nl);
      });
      if (s != ES_OK) return s;
    }
    if (!st.empty()) {
      s = h->timed(ES_KERNEL_STASH, sbytes, cs, [&](int *nl) {
        return es::launch_stash_multi((es_dtype)dd, (es_dtype)dd, st.data(), (int)st.size(), cs, h->blocks_ov,
                                      h->threads_ov, nl);
      });
      if (s != ES_OK) return s;
    }
  }
  for (int32_t i = 0; i < n; ++i) {
    const size_t k = (size_t)li * h->B + buckets[i];
    h->borrowed[k] = mode == ES_STASH_BORROW ? grads[i] : nullptr;
    if (cudaEventRecord(h->stash_ev[k], cs) != cudaSuccess) return h->poison(ES_ECUDA, "cudaEventRecord failed");
    h->stash_cap[k] = cap;
    h->stashed[k] = 1;
    h->inc_next[buckets[i]] = est + 1;
  }
  return ES_OK;
}

es_status es_stash_and_switch(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                              const es_dtype *gdts, es_stash_mode mode, int32_t next_est, es_stream stream) {
  if (next_est < 0) return set_err(ES_EINVAL, "next_est must be a valid EST (use es_stash_grads to only stash)");
  return stash_impl(h, est, n, buckets, grads, gdts, mode, next_est, stream);
}

es_status es_stash_grad(es_handle h, int32_t est, int32_t bucket, const void *grad, es_dtype gdt, es_stash_mode mode,
                        es_stream stream) {
  return stash_impl(h, est, 1, &bucket, &grad, &gdt, mode, -1, stream);
}

// ---- aggregation --------------------------------------------------------------------

namespace {
es_status finish_allreduce(es_handle h, int32_t n, const int32_t *buckets, cudaStream_t cs, unsigned long long cap);

es_status peer_barrier(es_handle h, cudaStream_t cs) {
  const es::Plan &p = h->plan;
  std::vector<uint64_t *> pf(p.G);
  for (int32_t g = 0; g < p.G; ++g) pf[g] = reinterpret_cast<uint64_t *>(h->peer_ws[g] + p.flags_off);
  const uint64_t epoch = ++h->barrier_epoch;
  return h->timed(ES_KERNEL_BARRIER, 0, cs, [&](int *nl) {
    *nl = 1;
    return es::launch_peer_barrier(pf.data(), reinterpret_cast<uint64_t *>(h->ws + p.flags_off), p.G, p.rank, epoch,
                                   cs);
  });
}

// ES_SCHED_PEER, phase-merged over the batch: [peer-visible copies of
// borrowed buckets] -> barrier -> one fold launch (own shards, remote
// contributions read from the owners' slots over NVLink) -> barrier -> one
// gather launch per dtype (every shard from its owner's RESULT area).
es_status peer_allreduce(es_handle h, int32_t n, const int32_t *buckets, void *const *outs, cudaStream_t cs, float r) {
  const es::Plan &p = h->plan;
  if (!h->peer_open) return set_err(ES_ESTATE, "ES_SCHED_PEER needs es_peer_open before es_allreduce");
  es_status s;
  const int32_t g = p.rank;
  auto slot_of = [&](int32_t rank, int32_t e, int32_t b) {
    return h->peer_ws[rank] + p.grad_off + (uint64_t)p.owner_index[e] * p.slot_block + p.slot_off[b];
  };
  // 1. borrowed contributions: peers read the ranges outside our shard from the slot
  for (int dd = 0; dd < 2; ++dd) {
    std::vector<es::StashSegDesc> segs;
    uint64_t nbytes = 0;
    for (int32_t i = 0; i < n; ++i) {
      const es::BucketPlan &b = p.bp[buckets[i]];
      if ((int)b.dtype != dd || b.L == 0) continue;
      for (int32_t li = 0; li < h->n_local; ++li) {
        const void *bw = h->borrowed[(size_t)li * h->B + buckets[i]];
        if (!bw) continue;
        unsigned char *slot = h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[buckets[i]];
        const unsigned char *src = reinterpret_cast<const unsigned char *>(bw);
        if (b.shard_lo > 0) segs.push_back({src, slot, b.shard_lo});
        if ((uint64_t)b.shard_hi < b.L)
          segs.push_back({src + (uint64_t)b.shard_hi * b.esize, slot + (uint64_t)b.shard_hi * b.esize,
                          (int64_t)(b.L - (uint64_t)b.shard_hi)});
        nbytes += 2 * (b.L - (uint64_t)(b.shard_hi - b.shard_lo)) * b.esize;
      }
    }
    if (segs.empty()) continue;
    s = h->timed(ES_KERNEL_STASH, nbytes, cs, [&](int *nl) {
      return es::launch_stash_multi((es_dtype)dd, (es_dtype)dd, segs.data(), (int)segs.size(), cs, h->blocks_ov,
                                    h->threads_ov, nl);
    });
    if (s != ES_OK) return s;
  }
  // 2. every rank's slots hold this step's contributions
  if ((s = peer_barrier(h, cs)) != ES_OK) return s;
  // 3. fold of the own shards
  for (int dd = 0; dd < 2; ++dd) {
    std::vector<es::FoldSegDesc> segs;
    std::vector<std::vector<const void *>> srcs;
    uint64_t nbytes = 0;
    for (int32_t i = 0; i < n; ++i) {
      const int32_t bk = buckets[i];
      const es::BucketPlan &b = p.bp[bk];
      if ((int)b.dtype != dd || b.shard_hi <= b.shard_lo) continue;
      std::vector<const void *> src(p.N);
      for (int32_t e = 0; e < p.N; ++e) {
        const int32_t li = p.local_index[e];
        const void *bw = li >= 0 ? h->borrowed[(size_t)li * h->B + bk] : nullptr;
        const unsigned char *base = bw ? reinterpret_cast<const unsigned char *>(bw) : slot_of(p.est_to_gpu[e], e, bk);
        src[e] = base + (uint64_t)b.shard_lo * b.esize;
      }
      es::FoldSegDesc d;
      d.lo = b.shard_lo;
      d.n = b.shard_hi - b.shard_lo;
      d.C = (uint32_t)b.C;
      d.rot = true;
      d.out = h->ws + p.result_off + p.slot_off[bk] + (uint64_t)b.shard_lo * b.esize;
      nbytes += (uint64_t)d.n * ((uint64_t)p.N + 1) * b.esize;
      segs.push_back(d);
      srcs.push_back(std::move(src));
    }
    if (segs.empty()) continue;
    for (size_t i = 0; i < segs.size(); ++i) segs[i].src = srcs[i].data();
    s = h->timed(ES_KERNEL_FOLD, nbytes, cs, [&](int *nl) {
      return es::launch_fold_multi((es_dtype)dd, p.N, r, p.compat, segs.data(), (int)segs.size(), cs, h->blocks_ov,
                                   h->threads_ov, nl);
    });
    if (s != ES_OK) return s;
  }
  // 4. every shard result is ready; every slot has been read
  if ((s = peer_barrier(h, cs)) != ES_OK) return s;
  // 5. gather every shard from its owner
  for (int dd = 0; dd < 2; ++dd) {
    std::vector<es::StashSegDesc> segs;
    uint64_t nbytes = 0;
    for (int32_t i = 0; i < n; ++i) {
      const int32_t bk = buckets[i];
      const es::BucketPlan &b = p.bp[bk];
      if ((int)b.dtype != dd || b.L == 0) continue;
      unsigned char *outp = reinterpret_cast<unsigned char *>(outs[i]);
      const uint64_t S = es::chunk_elems(b.L, p.G, p.A);
      for (int32_t o = 0; o < p.G; ++o) {
        const uint64_t lo = std::min<uint64_t>(b.L, S * o), hi = std::min<uint64_t>(b.L, S * (o + 1));
        if (hi <= lo) continue;
        segs.push_back({h->peer_ws[o] + p.result_off + p.slot_off[bk] + lo * b.esize, outp + lo * b.esize,
                        (int64_t)(hi - lo)});
        nbytes += 2 * (hi - lo) * b.esize;
      }
    }
    if (segs.empty()) continue;
    s = h->timed(ES_KERNEL_GATHER, nbytes, cs, [&](int *nl) {
      return es::launch_stash_multi((es_dtype)dd, (es_dtype)dd, segs.data(), (int)segs.size(), cs, h->blocks_ov,
                                    h->threads_ov, nl);
    });
    if (s != ES_OK) return s;
  }
  (void)g;
  return ES_OK;
}
}  // namespace

es_status es_allreduce_many(es_handle h, int32_t n, const int32_t *buckets, void *const *outs, es_stream stream) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (n < 0 || (n > 0 && (!buckets || !outs))) return set_err(ES_EINVAL, "bad bucket/out arrays");
  for (int32_t i = 0; i < n; ++i) {
    const int32_t bk = buckets[i];
    if (bk < 0 || bk >= h->B) return set_err(ES_EINVAL, "bucket out of range");
    for (int32_t j = 0; j < i; ++j)
      if (buckets[j] == bk) return set_err(ES_EINVAL, "bucket listed twice");
    const es::BucketPlan &b = p.bp[bk];
    if (b.L == 0) continue;
    if (!outs[i] || !aligned16(outs[i])) return set_err(ES_EINVAL, "out must be a 16-byte aligned device pointer");
    const unsigned char *o = reinterpret_cast<const unsigned char *>(outs[i]);
    if (o < h->ws + h->ws_bytes && h->ws < o + b.L * b.esize) return set_err(ES_EINVAL, "out overlaps the workspace");
    for (int32_t li = 0; li < h->n_local; ++li)
      if (!h->stashed[(size_t)li * h->B + bk])
        return set_err(ES_ESTATE, "es_allreduce before every local EST stashed this bucket");
  }
  for (int32_t i = 0; i < n; ++i) {
    for (int32_t li = 0; li < h->n_local; ++li)
      if (!h->stashed[(size_t)li * h->B + buckets[i]])
        return set_err(ES_ESTATE, "es_allreduce before every local EST stashed this bucket");
    if (h->inc_next[buckets[i]] != 0 && h->inc_next[buckets[i]] != p.N)
      return set_err(ES_ESTATE, "incremental fold of this bucket is incomplete");
  }
  cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
  const unsigned long long cap = capture_id(cs);
  for (int32_t i = 0; i < n; ++i)
    for (int32_t li = 0; li < h->n_local; ++li) {
      const size_t k = (size_t)li * h->B + buckets[i];
      if (h->stash_cap[k] == cap && cudaStreamWaitEvent(cs, h->stash_ev[k], 0) != cudaSuccess)
        return h->poison(ES_ECUDA, "cudaStreamWaitEvent failed");
    }
  if (h->last_ar && h->last_ar_cap == cap && cudaStreamWaitEvent(cs, h->last_ar, 0) != cudaSuccess)
    return h->poison(ES_ECUDA, "cudaStreamWaitEvent failed");

  const float r = 1.0f / (float)p.N;   // R5: fl32(1/N), correctly rounded fp32 division

  if (p.peer) {
    if ((s = peer_allreduce(h, n, buckets, outs, cs, r)) != ES_OK) return s;
    return finish_allreduce(h, n, buckets, cs, cap);
  }

  // Pending FOLD ops: consecutive folds (across buckets for G == 1, within a
  // chain round for G > 1) are independent and go out as one multi-segment
  // launch; a transport group flushes them first.
  std::vector<es::FoldSegDesc> pend;
  std::vector<std::vector<const void *>> pend_src;
  es_dtype pend_dt = ES_F32;
  uint64_t pend_bytes = 0;
  auto flush = [&]() -> es_status {
    if (pend.empty()) return ES_OK;
    for (size_t i = 0; i < pend.size(); ++i) pend[i].src = pend_src[i].data();
    es_status st = h->timed(ES_KERNEL_FOLD, pend_bytes, cs, [&](int *nl) {
      return es::launch_fold_multi(pend_dt, p.N, r, p.compat, pend.data(), (int)pend.size(), cs, h->blocks_ov,
                                   h->threads_ov, nl);
    });
    pend.clear();
    pend_src.clear();
    pend_bytes = 0;
    return st;
  };

  for (int32_t i = 0; i < n; ++i) {
    const int32_t bucket = buckets[i];
    const es::BucketPlan &b = p.bp[bucket];
    const uint32_t esz = b.esize;
    auto src_base = [&](int32_t e) -> unsigned char * {   // element 0 of local EST e's contribution
      const int32_t li = p.local_index[e];
      const void *bw = h->borrowed[(size_t)li * h->B + bucket];
      if (bw) return reinterpret_cast<unsigned char *>(const_cast<void *>(bw));
      return h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[bucket];
    };
    auto contrib_at = [&](int32_t e, int64_t lo) -> unsigned char * {
      if (p.local_index[e] >= 0) return src_base(e) + (uint64_t)lo * esz;
      return h->ws + p.stage_off + (uint64_t)b.stage_index[e] * b.stage_stride + (uint64_t)(lo - b.shard_lo) * esz;
    };
    auto part_at = [&](int64_t id, int64_t lo) -> unsigned char * {
      const es::Part &pt = b.parts[id];
      return h->ws + p.parts_off + pt.off + (uint64_t)(lo - pt.lo) * 4;
    };
    unsigned char *outp = reinterpret_cast<unsigned char *>(outs[i]);
    if (h->inc_next[bucket] == p.N && b.L > 0) {
      // NEXT-1 end of step: chunk c < N-1 continues from its partial (ESTs
      // c+1..N-1) over the stashed ESTs 0..c; chunk N-1 folds 0..N-1.
      if (!pend.empty() && pend_dt != b.dtype && (s = flush()) != ES_OK) return s;
      pend_dt = b.dtype;
      const float *part = reinterpret_cast<const float *>(h->ws + p.inc_off + p.inc_bucket_off[bucket]);
      for (int32_t c = 0; c < p.N; ++c) {
        const int64_t lo = std::min<int64_t>((int64_t)b.L, (int64_t)c * (int64_t)b.C);
        const int64_t hi = std::min<int64_t>((int64_t)b.L, (int64_t)(c + 1) * (int64_t)b.C);
        if (hi <= lo) continue;
        es::FoldSegDesc d;
        d.lo = lo;
        d.n = hi - lo;
        d.C = (uint32_t)b.C;
        d.rot = false;
        const bool cont = c < p.N - 1;
        d.m = cont ? c + 1 : p.N;
        d.part_in = cont ? part + lo : nullptr;
        d.out = outp + (uint64_t)lo * esz;
        std::vector<const void *> src;
        for (int32_t e = 0; e < d.m; ++e) src.push_back(src_base(e) + (uint64_t)lo * esz);
        pend_bytes += (uint64_t)d.n * ((uint64_t)d.m * esz + (cont ? 4 : 0) + esz);
        pend.push_back(d);
        pend_src.push_back(std::move(src));
      }
      continue;
    }
    for (const es::Op &op : b.ops) {
      const int64_t *f = op.f;
      switch (f[0]) {
        case ES_OP_FOLD: {
          if (!pend.empty() && pend_dt != b.dtype && (s = flush()) != ES_OK) return s;
          pend_dt = b.dtype;
          const int64_t lo = f[1], hi = f[2];
          es::FoldSegDesc d;
          d.lo = lo;
          d.n = hi - lo;
          d.C = (uint32_t)b.C;
          std::vector<const void *> src;
          if (f[3] < 0) {
            d.rot = true;
            for (int32_t e = 0; e < p.N; ++e) src.push_back(contrib_at(e, lo));
          } else {
            d.rot = false;
            d.m = (int32_t)f[4];
            for (int32_t t = 0; t < d.m; ++t) src.push_back(contrib_at((int32_t)((f[3] + t) % p.N), lo));
          }
          d.part_in = f[5] == ES_BUF_PART ? reinterpret_cast<const float *>(part_at(f[6], lo)) : nullptr;
          d.out_partial = f[7] == ES_BUF_PART;
          d.out = d.out_partial ? (void *)part_at(f[8], lo) : (void *)(outp + (uint64_t)lo * esz);
          pend_bytes += (uint64_t)d.n * ((uint64_t)src.size() * esz + (d.part_in ? 4 : 0) + (d.out_partial ? 4 : esz));
          pend.push_back(d);
          pend_src.push_back(std::move(src));
          break;
        }
        case ES_OP_GROUP_BEGIN:
          if ((s = flush()) != ES_OK) return s;
          if ((s = h->tp->group_begin()) != ES_OK) return h->poison(s, h->tp->err);
          break;
        case ES_OP_GROUP_END:
          if ((s = h->tp->group_end(cs)) != ES_OK) return h->poison(s, h->tp->err);
          break;
        case ES_OP_SEND:
        case ES_OP_RECV: {
          const int64_t lo = f[1], hi = f[2];
          const int peer = (int)f[3];
          unsigned char *ptr = nullptr;
          uint64_t w = esz;
          switch (f[4]) {
            case ES_BUF_SRC:
            case ES_BUF_STAGE: ptr = contrib_at((int32_t)f[5], lo); break;
            case ES_BUF_PART: ptr = part_at(f[5], lo); w = 4; break;
            case ES_BUF_OUT: ptr = outp + (uint64_t)lo * esz; break;
            default: return h->poison(ES_ESTATE, "corrupt plan: bad buffer kind");
          }
          const size_t nbytes = (size_t)(hi - lo) * w;
          s = f[0] == ES_OP_SEND ? h->tp->send(ptr, nbytes, peer) : h->tp->recv(ptr, nbytes, peer);
          if (s != ES_OK) return h->poison(s, h->tp->err);
          break;
        }
        default:
          return h->poison(ES_ESTATE, "corrupt plan: bad opcode");
      }
    }
  }
  if ((s = flush()) != ES_OK) return s;
  return finish_allreduce(h, n, buckets, cs, cap);
}

namespace {

es_status finish_allreduce(es_handle h, int32_t n, const int32_t *buckets, cudaStream_t cs, unsigned long long cap) {
  for (int32_t i = 0; i < n; ++i) {
    const int32_t bucket = buckets[i];
    if (cudaEventRecord(h->ar_ev[bucket], cs) != cudaSuccess) return h->poison(ES_ECUDA, "cudaEventRecord failed");
    h->ar_recorded[bucket] = 1;
    h->ar_cap[bucket] = cap;
    h->last_ar = h->ar_ev[bucket];
    h->last_ar_cap = cap;
    for (int32_t li = 0; li < h->n_local; ++li) {
      h->stashed[(size_t)li * h->B + bucket] = 0;
      h->borrowed[(size_t)li * h->B + bucket] = nullptr;
    }
    h->inc_next[bucket] = 0;
  }
  return ES_OK;
}

}  // namespace

es_status es_allreduce(es_handle h, int32_t bucket, void *out, es_stream stream) {
  return es_allreduce_many(h, 1, &bucket, &out, stream);
}

// ---- peer memory ---------------------------------------------------------------------

namespace {

struct PeerBlob {
  char magic[8];            // "ESPEER01"
  int32_t rank, pid;
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

}  // namespace

es_status es_peer_blob(es_handle h, void *blob, size_t bytes) {
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  if (!blob || bytes < ES_PEER_BLOB_BYTES) return set_err(ES_EINVAL, "blob must hold ES_PEER_BLOB_BYTES");
  PeerBlob b;
  std::memset(&b, 0, sizeof b);
  std::memcpy(b.magic, "ESPEER01", 8);
  b.rank = h->plan.rank;
  b.pid = (int32_t)getpid();
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
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (!blobs || bytes < (size_t)p.G * ES_PEER_BLOB_BYTES) return set_err(ES_EINVAL, "need G blobs");
  if (h->peer_open) return set_err(ES_ESTATE, "peers already open");
  std::vector<unsigned char *> ws(p.G, nullptr);
  std::vector<void *> mapped;
  const int32_t me = (int32_t)getpid();
  for (int32_t g = 0; g < p.G; ++g) {
    PeerBlob b;
    std::memcpy(&b, reinterpret_cast<const unsigned char *>(blobs) + (size_t)g * ES_PEER_BLOB_BYTES, sizeof b);
    if (std::memcmp(b.magic, "ESPEER01", 8) != 0 || b.rank != g) {
      for (void *m : mapped) cudaIpcCloseMemHandle(m);
      return set_err(ES_EINVAL, "blob g is not rank g's es_peer_blob");
    }
    int32_t n_g = 0;
    for (int32_t e = 0; e < p.N; ++e) n_g += p.est_to_gpu[e] == g;
    if (b.ws_bytes < p.grad_off + (uint64_t)n_g * p.slot_block) {
      for (void *m : mapped) cudaIpcCloseMemHandle(m);
      return set_err(ES_EINVAL, "peer workspace smaller than this layout");
    }
    if (g == p.rank) {
      ws[g] = h->ws;
    } else if (b.pid == me) {
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

// ---- instrumentation ---------------------------------------------------------

es_status es_profile_enable(es_handle h, int32_t on) {
  if (!h) return set_err(ES_EINVAL, "handle is NULL");
  h->prof = on != 0;
  return ES_OK;
}

static void drain(es_handle h) {
  for (auto &r : h->recs) {
    float t = 0.f;
    cudaEventSynchronize(r.b);
    cudaEventElapsedTime(&t, r.a, r.b);
    h->ms[r.kind] += t;
    std::vector<cudaEvent_t> &dst = r.captured ? h->graph_events : h->pool;
    dst.push_back(r.a);
    dst.push_back(r.b);
  }
  h->recs.clear();
}

es_status es_profile_reset(es_handle h) {
  if (!h) return set_err(ES_EINVAL, "handle is NULL");
  drain(h);
  for (int k = 0; k < ES_KERNEL_KINDS; ++k) {
    h->launches[k] = 0;
    h->bytes[k] = 0;
    h->ms[k] = 0;
  }
  return ES_OK;
}

es_status es_profile_query(es_handle h, es_kernel_kind kind, uint64_t *launches, double *ms, uint64_t *bytes) {
  if (!h) return set_err(ES_EINVAL, "handle is NULL");
  if (kind < 0 || kind >= ES_KERNEL_KINDS) return set_err(ES_EINVAL, "bad kernel kind");
  drain(h);
  if (launches) *launches = h->launches[kind];
  if (ms) *ms = h->ms[kind];
  if (bytes) *bytes = h->bytes[kind];
  return ES_OK;
}

es_status es_set_launch_override(es_handle h, int32_t blocks, int32_t threads) {
  if (!h) return set_err(ES_EINVAL, "handle is NULL");
  if (blocks < 0 || threads < 0 || threads > 256 || (threads % 32) != 0)
    return set_err(ES_EINVAL, "threads must be a multiple of 32 in [0, 256]; blocks >= 0");
  h->blocks_ov = blocks;
  h->threads_ov = threads;
  return ES_OK;
}

}  // extern "C"
