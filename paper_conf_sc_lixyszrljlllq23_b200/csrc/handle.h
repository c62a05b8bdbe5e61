// handle.h -- the per-rank handle of libes (es_ctx) and the helpers every
// C-ABI translation unit shares: thread-local error detail, sticky errors,
// CUDA-graph capture ids, launch timing (internal).
#pragma once

#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <cstring>
#include <memory>
#include <string>
#include <vector>

#include "../../include/es.h"
#include "kernels.h"
#include "plan.h"
#include "transport.h"

namespace es_detail {

extern thread_local std::string g_err;

inline es_status set_err(es_status s, const std::string &msg) {
  g_err = msg;
  return s;
}

// Tracing: one NVTX range per C-ABI call that enqueues work, named after the call, so
// nsys timelines and `ncu --nvtx` filters see the stash / switch / allreduce structure of a step.
// NVTX v3 is header-only; without an attached tool a range costs one predictable branch.
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange &) = delete;
  NvtxRange &operator=(const NvtxRange &) = delete;
};
#define ES_NVTX() ::es_detail::NvtxRange es_nvtx_range_(__func__)

inline bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// CUDA-graph support: the id of the capture `s` is part of, 0 when eager.
// Events recorded in one capture (or eagerly) are only waited on from the
// same capture (or eagerly): a graph cannot depend on work outside it, and
// replays of a graph on one stream are ordered anyway.
inline unsigned long long capture_id(cudaStream_t s) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  unsigned long long id = 0;
  if (cudaStreamGetCaptureInfo(s, &st, &id) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return st == cudaStreamCaptureStatusActive ? id : 0;
}

}  // namespace es_detail

using es_detail::set_err;
using es_detail::aligned16;
using es_detail::capture_id;

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

  // graph capture: node of our last stash launch (early-start proof)
  cudaGraphNode_t last_stash_node = nullptr;
  unsigned long long last_stash_cap = 0;

  // NEXT-1 incremental fold: next EST expected per bucket (0: none folded yet)
  std::vector<int32_t> inc_next;
  // [local EST index * B + bucket]: 1 if an incremental COPY stash left the EST's
  // whole gradient in the slot (exportable), 0 if part of it lives only in the partials
  std::vector<uint8_t> inc_full;

  // ES_SCHED_PEER
  std::vector<unsigned char *> peer_ws;   // [G] workspace base of every rank, mapped here
  std::vector<void *> ipc_mapped;         // cudaIpcOpenMemHandle results to close
  bool peer_open = false;
  int32_t peer_share = 1;                 // ranks of this process sharing the device (loopback)

  // CHAIN over a transport, tile-pipelined: the partials' transfers run on this
  // library-owned stream (created on first use), ordered against the caller's
  // stream with events, so they overlap later tiles' folds.
  cudaStream_t side = nullptr;
  std::vector<cudaEvent_t> chain_ev;      // ordering events of chain_pipelined (reused per call)

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
  // ES_OPT_STASH_BACKGROUND: same-dtype stashes run as the small TMA ring
  // (launch_stash_multi); the other switch-time kernels (casts, incremental
  // folds) get a grid capped (negative = a cap for the launchers) at two
  // 256-thread CTAs per SM, so the model's kernels queued behind them are
  // dispatched at once ("Overlap with compute").
  bool background() const { return (plan.options & ES_OPT_STASH_BACKGROUND) != 0; }
  int switch_blocks() const {
    return blocks_ov ? blocks_ov : ((plan.options & ES_OPT_STASH_BACKGROUND) ? -2 * 148 : 0);
  }
  int switch_threads() const { return threads_ov ? threads_ov : ((plan.options & ES_OPT_STASH_BACKGROUND) ? 256 : 0); }

  ~es_ctx() {
    for (auto e : stash_ev) if (e) cudaEventDestroy(e);
    for (auto e : ar_ev) if (e) cudaEventDestroy(e);
    for (auto &r : recs) { cudaEventDestroy(r.a); cudaEventDestroy(r.b); }
    for (auto e : pool) cudaEventDestroy(e);
    for (auto e : graph_events) cudaEventDestroy(e);
    for (void *p : ipc_mapped) cudaIpcCloseMemHandle(p);
    for (auto e : chain_ev) cudaEventDestroy(e);
    if (side) cudaStreamDestroy(side);
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

inline es_status check_handle(es_handle h) {
  if (!h) return set_err(ES_EINVAL, "handle is NULL");
  return h->check_sticky();
}

// Early start of a stash kernel is safe only when the kernel immediately
// before it on the stream is one of our own stash or switch kernels
// (independent data; the fused swap blocks still wait).  That is provable only inside a CUDA-graph capture: the stream's
// capture dependencies must be exactly the node of our previous stash launch
// (no foreign kernel, event wait or timing node in between).  Eager launches
// never start early.
inline bool follows_own_stash(es_handle h, cudaStream_t cs) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  unsigned long long id = 0;
  cudaGraph_t g = nullptr;
  const cudaGraphNode_t *deps = nullptr;
  size_t nd = 0;
  if (cudaStreamGetCaptureInfo(cs, &st, &id, &g, &deps, &nd) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return st == cudaStreamCaptureStatusActive && nd == 1 && h->last_stash_node && deps[0] == h->last_stash_node &&
         id == h->last_stash_cap;
}

inline void remember_stash_node(es_handle h, cudaStream_t cs) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  unsigned long long id = 0;
  cudaGraph_t g = nullptr;
  const cudaGraphNode_t *deps = nullptr;
  size_t nd = 0;
  h->last_stash_node = nullptr;
  if (cudaStreamGetCaptureInfo(cs, &st, &id, &g, &deps, &nd) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  if (st == cudaStreamCaptureStatusActive && nd == 1 && !h->prof) {
    h->last_stash_node = deps[0];
    h->last_stash_cap = id;
  }
}
