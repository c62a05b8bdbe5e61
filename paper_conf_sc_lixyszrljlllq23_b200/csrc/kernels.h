// kernels.h -- launchers of the sm_100a kernels of libes (internal).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/es.h"

namespace es {

// One independent fold range over the
// bucket elements [lo, lo+n).  Every pointer points at element `lo` of its
// buffer (physical pointers, 16-byte aligned); lo must be a multiple of 8 so
// that no 16-byte vector straddles a chunk (R1 with A % 8 == 0).
//   rot == true : per-element canonical rotation -- element i = lo+t lies in
//                 chunk c = i / C and is folded over src[(c+1)%N], ...,
//                 src[(c+N)%N]  (src holds N pointers indexed by EST)
//   rot == false: sources src[0], ..., src[m-1] in that order (one chain
//                 segment, already in canonical order)
//   part_in     : if non-null, the fold continues from this unrounded fp32
//                 partial (R14) instead of starting from its first source
//   out_partial : write the unrounded fp32 sum to `out` (fp32); otherwise
//                 write round_dtype(fl32(s * r)) to `out` (bucket dtype).
struct FoldSegDesc {
  int64_t lo = 0, n = 0;
  uint32_t C = 1;
  bool rot = true;
  int32_t m = 0;
  const void *const *src = nullptr;   // host array: N (rot) or m pointers
  const float *part_in = nullptr;
  void *out = nullptr;
  bool out_partial = false;
  void *const *push = nullptr;        // ES_OPT_PEER_PUSH: npush more destinations of the final result
  int32_t npush = 0;
};

// Folds all segments (same dtype, same N) with as few launches as the
// parameter capacity allows (one for every configuration this build plans
// for up to 64 segments and 1024 source pointers).  *launches receives the
// number of kernels enqueued.
// compat: NEXT-3 variant bits (ES_COMPAT_*); 0 = the canonical definition.
cudaError_t launch_fold_multi(es_dtype dtype, int32_t N, float r, uint32_t compat, const FoldSegDesc *segs, int nseg,
                              cudaStream_t s, int blocks_override, int threads_override, int *launches);

// PEER_CHAIN, tile-pipelined (k_fold_pipe): chain segments (rot == false)
// cut into tiles of kPipeTile elements.  wait: the producer GPU's flags of
// this chunk's previous round (tile t at wait[t]; null in round 0); pub: this
// GPU's flags of the round (null when the chunk ends here).  Segments must be
// passed in round-major order.  epoch: this rank's barrier epoch word (the
// flag value is *epoch + 1); ticket: a zeroable device word; share: number of
// ranks sharing this device (the grid is cut so that all of them fit).
constexpr int kPipeTile = 8192;
struct PipeSegDesc {
  FoldSegDesc f;
  const uint64_t *wait = nullptr;
  uint64_t *pub = nullptr;
};
cudaError_t launch_fold_pipe(es_dtype dtype, int32_t N, float r, const PipeSegDesc *segs, int nseg,
                             const uint64_t *epoch, unsigned int *ticket, int share, cudaStream_t s, int *launches);

// Stash segments: dst[i] = cast(src[i]) for i < n, all with
// the same (source dtype, destination dtype).
struct StashSegDesc {
  const void *src;
  void *dst;
  int64_t n;
};
// Context-switch swap table entry.
struct SwapEntry {
  unsigned char *live;   // live buffer (16-byte aligned)
  unsigned char *slot0;  // saved copy of local EST 0; local EST k at slot0 + k*stride
  uint64_t stride;
  uint64_t nbytes;
};

// A context swap to fuse into a stash launch (n == 0: none).
struct SwapArgs {
  const SwapEntry *tab = nullptr;
  int32_t n = 0;
  uint64_t max_nbytes = 0;
  int32_t cur = -1, next = 0;
};

// If `swap` has entries, its blocks ride in the first stash launch (the
// outgoing EST's stash and the context switch are independent), saving one
// launch per context switch.
// early: the caller has proven that the kernel immediately preceding this
// launch on `s` is one of our stash kernels (independent data), so the copy
// blocks may start while it is still running -- they wait for it only before
// exiting (completion order stays transitive); swap blocks always wait first.
cudaError_t launch_stash_multi(es_dtype sdt, es_dtype ddt, const StashSegDesc *segs, int nseg, cudaStream_t s,
                               int blocks_override, int threads_override, int *launches,
                               const SwapArgs *swap = nullptr, bool early = false, bool background = false);

// One launch: for every entry, slot[cur] <- live, live <- slot[next]
// (cur < 0: load only).  max_nbytes sizes the grid.
cudaError_t launch_swap(const SwapEntry *table_dev, int32_t n, uint64_t max_nbytes, int32_t cur, int32_t next,
                        cudaStream_t s);

// NEXT-4 per-EST dropout: y = dropout(x, p)
// driven by the Philox record {seed u64, offset u64} at `record` (the live
// context buffer of the running EST); the kernel advances record.offset by
// one when the whole grid has read it (`counter`: a zeroed u32 in the
// workspace).  x / y 16-byte aligned; mask (nullable) gets 1 = kept.
cudaError_t launch_dropout(es_dtype dtype, const void *x, void *y, uint8_t *mask, int64_t n, float p, float scale,
                           uint64_t *record, unsigned int *counter, cudaStream_t s);

// PEER barrier: the epoch e = my_flags[kEpochSlot] + 1 lives in device memory
// (so a CUDA-graph replay advances it); thread t < G publishes e into slot
// `rank` of peer t's flag array (system-scope release) and then waits until
// this rank's own flag array holds >= e in every slot (system-scope acquire).
// One block.  my_flags has kPeerFlagWords u64 words, zeroed at es_init.
constexpr int kEpochSlot = 64;
constexpr int kTicketSlot = 65;     // k_fold_pipe's work counter (local)
constexpr int kPeerFlagWords = 66;
cudaError_t launch_peer_barrier(uint64_t *const *peer_flags, uint64_t *my_flags, int32_t G, int32_t rank,
                                cudaStream_t s);

// Force-load every kernel instantiation libes can launch (see kernel_registry
// in kernels.cu); called before any device-side spin-wait can run.
cudaError_t preload_kernels();
size_t registered_kernels();

// Programmatic dependent launch (on by default; ES_NO_PDL=1 disables).
void set_pdl(bool on);

}  // namespace es
