// api_core.cpp -- C ABI: versions and errors, sizing, plan export, handle lifetime,
// context state registration and the context switch, instrumentation.
#include <unistd.h>

#include "handle.h"

namespace es_detail {
thread_local std::string g_err;
}  // namespace es_detail

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

const char *es_last_error(void) { return es_detail::g_err.c_str(); }

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

es_status es_plan_incremental(const es_config *cfg, int32_t bucket, int64_t *rows, size_t cap_rows,
                              size_t *n_rows) {
  if (!n_rows) return set_err(ES_EINVAL, "n_rows is NULL");
  es::Plan p;
  std::string err;
  es_status s = es::build_plan(cfg, &p, &err, false);
  if (s != ES_OK) return set_err(s, err);
  if (bucket < 0 || bucket >= (int32_t)p.bp.size()) return set_err(ES_EINVAL, "bucket out of range");
  const es::BucketPlan &b = p.bp[bucket];
  *n_rows = b.inc.size();
  if (rows)
    for (size_t i = 0; i < b.inc.size() && i < cap_rows; ++i) {
      const es::IncChunk &ic = b.inc[i];
      const int64_t r[5] = {ic.c, ic.first, ic.q, ic.lo, ic.hi};
      std::memcpy(rows + 5 * i, r, sizeof r);
    }
  return ES_OK;
}

es_status es_init(const es_config *cfg, void *workspace, size_t workspace_bytes, es_handle *out) {
  ES_NVTX();
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
  h->inc_full.assign(nslot, 0);
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
  // The tile-pipelined CHAIN's side stream, created here rather than at its first use, which may
  // be inside a CUDA-graph capture.
  for (const es::BucketPlan &b : h->plan.bp)
    if (b.sched == ES_SCHED_CHAIN && !(h->plan.options & ES_OPT_PEER_ROUNDS) && !h->side &&
        cudaStreamCreateWithFlags(&h->side, cudaStreamNonBlocking) != cudaSuccess)
      return set_err(ES_ECUDA, "cudaStreamCreate failed");
  {
    // Zero the scratch words and the peer flags + epoch counter on a private
    // stream and wait for it: peers may write these flags as soon as they hold
    // this rank's peer blob, and other ranks' work on shared streams must not
    // be waited for (loopback ranks initialise concurrently).
    cudaStream_t zs = nullptr;
    if (cudaStreamCreateWithFlags(&zs, cudaStreamNonBlocking) != cudaSuccess)
      return set_err(ES_ECUDA, "cudaStreamCreate failed");
    bool ok = cudaMemsetAsync(h->ws + h->plan.scratch_off, 0, 256, zs) == cudaSuccess;
    if (ok && h->plan.peer) ok = cudaMemsetAsync(h->ws + h->plan.flags_off, 0, es::kPeerFlagWords * 8, zs) == cudaSuccess;
    if (ok && h->plan.pipe_flag_words > 0)
      ok = cudaMemsetAsync(h->ws + h->plan.pipe_flags_off, 0, h->plan.pipe_flag_words * 8, zs) == cudaSuccess;
    ok = cudaStreamSynchronize(zs) == cudaSuccess && ok;
    cudaStreamDestroy(zs);
    if (!ok) return set_err(ES_ECUDA, "cudaMemsetAsync of the workspace scratch / peer flags failed");
  }
  if (h->plan.G > 1 && h->plan.transport != ES_TRANSPORT_NONE) {
    es::Transport *t = h->plan.transport == ES_TRANSPORT_NCCL
                           ? es::make_nccl_transport(h->plan.comm, h->plan.G, h->plan.rank, &err)
                           : es::make_loopback_transport(h->plan.comm, h->plan.G, h->plan.rank, &err);
    if (!t) return set_err(h->plan.transport == ES_TRANSPORT_NCCL ? ES_ENCCL : ES_EINVAL, err);
    h->tp.reset(t);
  } else if (h->plan.transport == ES_TRANSPORT_NCCL && h->plan.comm) {
    // G == 1 needs no exchange, but a communicator that was passed must still
    // be a size-1 NCCL comm of this rank (catches a wrong pointer early).
    std::unique_ptr<es::Transport> t(es::make_nccl_transport(h->plan.comm, 1, h->plan.rank, &err));
    if (!t) return set_err(ES_ENCCL, err);
  }
  *out = h.release();
  return ES_OK;
}

es_status es_destroy(es_handle h) {
  ES_NVTX();
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
  ES_NVTX();
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
    remember_stash_node(h, cs);      // a following stash may start early (independent data)
  }
  h->cur_local = li;
  return ES_OK;
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
    // A captured pair that was never replayed (or an eager pair that failed)
    // has no time: skip it and clear the error it raised, so it cannot
    // surface later as some other call's launch failure.
    if (cudaEventSynchronize(r.b) == cudaSuccess && cudaEventElapsedTime(&t, r.a, r.b) == cudaSuccess)
      h->ms[r.kind] += t;
    else
      cudaGetLastError();
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
