/*
 * es.h -- C ABI of libes, the B200-native placement-invariant EST gradient
 * aggregator (EasyScale, SC '23; PAPER.md = arXiv 2208.14228v3 text).
 *
 * "P:n" cites line n of PAPER.md; "Rn" cites a reading in DESIGN.md
 * ("Readings of the paper"), which fixes what the paper leaves unstated.
 *
 * The hot path (PAPER.md 3.2 "EasyScaleThread", and 3.3 "D1
 * elastic determinism"):
 *
 *   N logical EasyScaleThreads (ESTs) -- DDP workers with constant virtual
 *   ranks 0..N-1 -- are time-sliced onto G GPUs.
 *   At each EST's context switch its gradient buckets are stashed
 *   (es_stash_grad) and its RNG / BatchNorm context is swapped
 *   (es_switch_context).  After the last local EST the
 *   buckets are aggregated across all N ESTs (es_allreduce, P:526-532,
 *   P:963-967) in ONE canonical order that depends only on N, the persisted
 *   bucket layout and the chunk alignment A -- never on G or on the
 *   EST->GPU mapping -- so the result is bitwise identical for any placement
 *   (D1; readings R1-R6, R13):
 *
 *     C = A*ceil(ceil(L/N)/A);  element i lies in chunk c = floor(i/C);
 *     s = x[(c+1)%N][i];  for j = 2..N: s = fl32(s + x[(c+j)%N][i]);
 *     out[i] = round_to_bucket_dtype(fl32(s * fl32(1/N))).
 *
 * Conventions for every function:
 *   - extern "C", never throws, returns es_status (ES_OK == 0).
 *   - Pointers named *_dev / grad / out / workspace are CUDA device pointers
 *     (cudaMalloc / torch CUDA storage) on the calling thread's current
 *     device; host_* pointers are ordinary host memory.
 *   - Argument errors (ES_EINVAL) are detected synchronously and have no
 *     side effects.  Protocol errors return ES_ESTATE.  A CUDA / NCCL error
 *     at enqueue time returns ES_ECUDA / ES_ENCCL and poisons the handle:
 *     every later call on it returns the same status (sticky).
 *     Asynchronous device faults surface at es_sync().
 *   - es_last_error() returns a thread-local human-readable detail string
 *     for the most recent failing call on this thread.
 *   - A handle is not thread-safe; use one handle per thread (one per GPU
 *     rank).  Different handles may be used concurrently.
 *   - Every call that enqueues device work is an NVTX range named after the
 *     call ("es_stash_and_switch", "es_allreduce_many", ...) for nsys / ncu
 *     filtering (NVTX v3; a no-op when no tool is attached).
 */
#ifndef ES_H
#define ES_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ES_ABI_VERSION 1

typedef struct es_ctx *es_handle;        /* opaque; one per rank (= per GPU) */
typedef struct CUstream_st *es_stream;   /* identical to cudaStream_t; NULL = legacy default stream */

typedef enum {
  ES_OK = 0,
  ES_EINVAL = 1,        /* bad argument (synchronous, no side effects)            */
  ES_ESTATE = 2,        /* protocol violation (missing stash, non-local EST, ...)  */
  ES_ENOMEM = 3,        /* workspace too small                                     */
  ES_ECUDA = 4,         /* CUDA runtime error (sticky)                             */
  ES_ENCCL = 5,         /* NCCL error / NCCL library not loadable (sticky)         */
  ES_EUNSUPPORTED = 6   /* feature not available in this build / on this device   */
} es_status;

/* Element types.  A bucket's dtype is the dtype of its slots and of the
 * aggregated output; accumulation is always fp32 (R4). */
typedef enum { ES_F32 = 0, ES_BF16 = 1 } es_dtype;

/* ES_STASH_COPY copies (or casts) the gradient into the EST's slot in the
 * workspace; the caller may overwrite `grad` once `stream` has passed the
 * call.  ES_STASH_BORROW records the pointer only -- the paper's last local
 * EST, whose gradients are synchronised in place; the buffer
 * must stay unchanged until es_allreduce of that bucket has completed on
 * its stream, and must already hold the bucket dtype. */
/* ES_STASH_INPLACE: the gradient was produced directly in the EST's slot
 * (es_slot_ptr -- DDP bucket views bound to the slot);
 * `grad` must be that slot pointer; no kernel runs. */
typedef enum { ES_STASH_COPY = 0, ES_STASH_BORROW = 1, ES_STASH_INPLACE = 2 } es_stash_mode;

/* Exchange schedule for G > 1.  Both produce the
 * same bits; they differ only in NVLink bytes.
 *   DIRECT: GPU g owns element shard S_g, receives the N - n_g remote
 *           contributions for it, folds all N in canonical order, then the
 *           shards are all-gathered.
 *   CHAIN:  chunk c's unrounded fp32 partial walks the GPUs in canonical
 *           EST order; each GPU folds its consecutive local ESTs; the GPU of
 *           EST c scales, rounds and owns chunk c; then all-gather.  By
 *           default the rounds are tile-pipelined: every chunk is cut into
 *           the same number of tiles W (<= 8, ~2^20 elements each), the fold
 *           of (round r, tile w) runs on the caller's stream and the transfer
 *           of its partial on a library-owned side stream, ordered by events,
 *           in (r + w) wavefront order, so transfers overlap later tiles'
 *           folds; ES_OPT_PEER_ROUNDS keeps one fold launch + one transfer
 *           group per round (same bits, same messages per peer pair).
 *   AUTO:   per bucket, the one with fewer max-per-GPU received bytes
 *           (ties -> DIRECT).  The choice is identical on every rank. */
/*   PEER:   no transport library: rank g's fold kernel pulls the remote
 *           ESTs' contributions for its shard straight out of the peers'
 *           slots over NVLink (CUDA IPC-mapped workspaces, es_peer_*), writes
 *           its shard result into its own workspace, and a gather kernel pulls
 *           every other shard from its owner; device-side barriers (flags in
 *           peer memory) order the phases.  No staging copy, no NCCL protocol.
 *           Opt-in (never chosen by AUTO); BORROWed buckets are made
 *           peer-visible by copying the parts peers read into the slot. */
/*   PEER_CHAIN: the CHAIN schedule without a transport: the GPU of segment r
 *           of chunk c reads the incoming unrounded fp32 partial directly from
 *           the producer's workspace over NVLink inside its fold kernel (the
 *           partial's transfer and the local fold are one kernel).  By
 *           default all rounds run as ONE tile-pipelined kernel per dtype:
 *           the consumer of a partial starts on tile t as soon as the
 *           producer has published tile t (per-tile flags in peer memory), so
 *           the only device barriers are at the start and the end of the
 *           step; ES_OPT_PEER_ROUNDS runs one fold launch per round with a
 *           barrier between rounds instead (same bits).  Chunk c is gathered
 *           from the RESULT area of the GPU of EST c.
 *   PEER_AUTO: per bucket PEER_CHAIN where CHAIN would move fewer bytes,
 *           else PEER (the AUTO rule over the peer-memory schedules). */
typedef enum {
  ES_SCHED_AUTO = 0, ES_SCHED_DIRECT = 1, ES_SCHED_CHAIN = 2, ES_SCHED_PEER = 3, ES_SCHED_PEER_CHAIN = 4,
  ES_SCHED_PEER_AUTO = 5
} es_sched;

/* How ranks exchange bytes when G > 1.
 *   NONE:     G == 1, or G > 1 with sched PEER (no transport library needed).
 *   NCCL:     `comm` is a borrowed ncclComm_t over exactly the G ranks
 *             (e.g. torch ProcessGroupNCCL._comm_ptr()).  Only point-to-point
 *             ncclSend/ncclRecv inside ncclGroupStart/End are used -- never an
 *             NCCL reduction, whose order is not the canonical one.  libnccl is
 *             resolved at es_init from the copy already loaded in the process
 *             (dlopen RTLD_NOLOAD "libnccl.so.2"), else dlopen'ed by name.
 *             With G == 1 a non-NULL comm is only validated (size 1, rank 0;
 *             ES_ENCCL otherwise) and never used.
 *   LOOPBACK: `comm` is an es_loopback world (es_loopback_create); all G ranks
 *             live in ONE process, each driven by its own host thread, all
 *             on the same device; bytes move with cudaMemcpyAsync.  Test
 *             transport that lets a single GPU run every G and mapping. */
typedef enum { ES_TRANSPORT_NONE = 0, ES_TRANSPORT_NCCL = 1, ES_TRANSPORT_LOOPBACK = 2 } es_transport;

/* One DDP gradient bucket; its index in the array is the bucket id.  The
 * bucket layout is persisted state and part of the canonical definition
 * (R8, R9). */
typedef struct {
  uint64_t numel;       /* elements, < 2^31 */
  es_dtype dtype;
} es_bucket_desc;

typedef struct {
  int32_t N;                      /* logical ESTs, 1..1024                         */
  int32_t G;                      /* GPUs (ranks), 1..64, G <= N                               */
  int32_t rank;                   /* this process's GPU rank, 0..G-1                           */
  const int32_t *est_to_gpu;      /* host [N]: GPU of each EST; every GPU owns >= 1 EST (R10);
                                     identical on all ranks                                    */
  const es_bucket_desc *buckets;  /* host [n_buckets]: persisted layout (D1)                   */
  int32_t n_buckets;              /* 1..4096                                                   */
  uint32_t chunk_align;           /* A in elements; 0 => 16; must be a multiple of 8 (R1)      */
  int32_t n_state;                /* registered per-EST context buffers (Philox record, BN
                                     running stats), 0..4096            */
  const uint64_t *state_nbytes;   /* host [n_state]: bytes of each context buffer              */
  es_transport transport;
  void *comm;                     /* ncclComm_t (NCCL), es_loopback world (LOOPBACK), NULL (NONE) */
  es_sched sched;
  uint32_t compat;                /* 0 = the canonical definition (R1-R6, R13); else ES_COMPAT_*
                                     bits.  Part of the persisted definition. */
  uint32_t options;               /* ES_OPT_* bits (execution choices; never change bits)      */
} es_config;

/* ES_OPT_INCREMENTAL: reserve fp32 partials so that es_stash_fold_grads can
 * fold each EST into the running partials at its switch (NEXT-1, any G). */
#define ES_OPT_INCREMENTAL 1u
/* ES_OPT_PEER_ROUNDS: CHAIN and PEER_CHAIN without tile pipelining (PEER_CHAIN:
 * a device barrier between rounds; CHAIN: one fold launch and one transfer
 * group per round, one stream).  Same bits; kept for comparison and as a
 * fallback. */
#define ES_OPT_PEER_ROUNDS 2u
/* ES_OPT_STASH_BACKGROUND: stash for overlap with the model's compute
 * (PAPER.md:599-606).  A one-shot stash grid of thousands of CTAs is
 * dispatched ahead of any kernel queued after it on another stream, so the
 * next forward waits for the whole stash, and its CTAs take SM slots a GEMM
 * needs.  With this option same-dtype stashes run as one warp per SM driving
 * a 4 x 4 KB TMA bulk-copy ring (16 KB of shared memory: it fits beside a
 * tensor-core GEMM's CTA); casts, the fused context swap's launch and the
 * incremental folds use at most two 256-thread CTAs per SM.  About half the
 * copy bandwidth when nothing else runs.  Same bits. */
#define ES_OPT_STASH_BACKGROUND 4u
/* ES_OPT_PEER_PUSH (G > 1, ES_SCHED_PEER buckets, and ES_SCHED_PEER_CHAIN
 * buckets under ES_OPT_PEER_ROUNDS): the all-gather is fused
 * into the fold.  Each owner's fold writes its finished shard / chunk into
 * its own RESULT area AND into every peer's RESULT area over NVLink (posted
 * stores, riding the fold's egress while its ingress pulls the remote
 * contributions); after the barrier every rank copies the whole bucket from
 * its OWN RESULT area into `out` (local HBM) instead of pulling each shard
 * from its owner.  Same ops, same bits, same NVLink bytes per GPU: the other
 * shards arrive during the fold phase as their owners' posted stores instead
 * of during the gather as this rank's remote loads.  Ignored
 * (pull gather) when N + G - 1 > 1024. */
#define ES_OPT_PEER_PUSH 8u

/* NEXT-3 compatibility variants -- same canonical order, different step
 * arithmetic:
 *   PREDIV:   each contribution is divided by N first (PyTorch 1.8 DDP's
 *             div_ before the all-reduce); no post-scale.
 *   PREMUL:   each contribution is multiplied by fl32(1/N) first (NCCL
 *             ncclAvg / PreMulSum); no post-scale.  Exclusive with PREDIV.
 *   BF16_HOP: bf16 buckets only: every stored intermediate (scaled
 *             contribution, partial sum) is rounded to bf16, as an NCCL bf16
 *             ring stores it between hops.  Ignored for fp32 buckets. */
#define ES_COMPAT_PREDIV 1u
#define ES_COMPAT_PREMUL 2u
#define ES_COMPAT_BF16_HOP 4u

/* ---- sizing / lifetime --------------------------------------------------- */

/* Bytes of device workspace es_init needs for `cfg` (per-EST gradient and
 * context slots for the local ESTs, exchange staging, chain partials,
 * tables).  Host-only; no CUDA call.  ES_EINVAL on an invalid config. */
es_status es_workspace_bytes(const es_config *cfg, size_t *bytes);

/* Creates a handle.  `workspace` is caller-owned device memory of at least
 * es_workspace_bytes() bytes, 256-byte aligned, outliving the handle; the
 * library never calls cudaMalloc (PyTorch stays the only device allocator)
 * and owns only host metadata, CUDA events, for G > 1 its planner tables
 * and, when a CHAIN bucket runs tile-pipelined over a transport, one
 * non-blocking side stream (created here, destroyed by es_destroy).  The bucket plan (chunk table, shards, schedule, exchange ops) is
 * computed here once and never rebuilt (D1).  Elastic change of
 * G or of the mapping = es_destroy + es_init with the same N, layout and A
 * (P:619-624).  cfg and its arrays are copied. */
es_status es_init(const es_config *cfg, void *workspace, size_t workspace_bytes, es_handle *out);

/* Releases host resources.  Does not synchronise; the caller must not
 * destroy a handle with work still in flight (call es_sync first). */
es_status es_destroy(es_handle h);

/* Waits for all work this handle enqueued and reports asynchronous faults
 * (ES_ECUDA, sticky). */
es_status es_sync(es_handle h);

/* ---- EST context: stash + state swap ----------------------------------- */

/* Binds the live copies of the n == cfg.n_state context buffers (device
 * pointers, 16-byte aligned, sizes as in cfg.state_nbytes).  Must precede
 * es_switch_context when n_state > 0. */
es_status es_register_state(es_handle h, int32_t n, void *const *live_dev_ptrs);

/* Synchronously writes the saved copy of context buffer `idx` of local EST
 * `est` from host memory (state_nbytes[idx] bytes).  Used to seed each
 * EST's Philox record / BN statistics (D0: fixed seeds). */
es_status es_init_state(es_handle h, int32_t est, int32_t idx, const void *host_src);

/* Synchronously reads the saved copy of context buffer `idx` of local EST
 * `est` into host memory.  (The live copy belongs to the running EST.) */
es_status es_read_state(es_handle h, int32_t est, int32_t idx, void *host_dst);

/* Context switch to local EST `est` at a mini-batch boundary:
 * one kernel saves every live context buffer into the current EST's slot
 * and loads `est`'s slot into the live buffers.  The first switch only
 * loads.  Switching to the current EST is a no-op.  ES_ESTATE if `est` is
 * not mapped to this rank. */
es_status es_switch_context(es_handle h, int32_t est, es_stream stream);

/* Stashes local EST `est`'s gradient for `bucket`.
 * grad: device pointer, 16-byte aligned, `numel` elements of grad_dtype.
 * COPY: one vectorised kernel copies/casts into the EST's slot (RNE when
 * narrowing fp32->bf16, exact when widening); the copy waits (on `stream`)
 * for the bucket's previous es_allreduce, which may still read the slot.
 * BORROW: grad_dtype must equal the bucket dtype; the pointer is recorded.
 * INPLACE: grad must be es_slot_ptr(est, bucket); nothing is copied.  In
 * every mode an event on `stream` orders the stash before the bucket's
 * next es_allreduce.  ES_ESTATE if `est` is not mapped to this rank or the
 * bucket is being folded incrementally this step. */
es_status es_stash_grad(es_handle h, int32_t est, int32_t bucket, const void *grad,
                        es_dtype grad_dtype, es_stash_mode mode, es_stream stream);

/* Batched form of es_stash_grad: stashes n buckets of local EST `est` (the
 * paper swaps all of an EST's gradients at its context switch)
 * with one multi-segment kernel per (grad dtype, bucket dtype) pair.
 * buckets/grads/grad_dtypes are host arrays of length n; the same rules as
 * es_stash_grad apply to every entry; validation of all entries happens
 * before anything is enqueued. */
es_status es_stash_grads(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                         const es_dtype *grad_dtypes, es_stash_mode mode, es_stream stream);

/* The paper's context switch at a mini-batch boundary: stash
 * the outgoing local EST `est`'s gradients (n buckets, as es_stash_grads)
 * AND switch the RNG / BN context to local EST `next_est` (as
 * es_switch_context) with ONE kernel launch -- the two are independent, so
 * the swap blocks ride along in the stash grid.  Equivalent to
 * es_stash_grads(...) followed by es_switch_context(next_est).  next_est must
 * be a valid local EST (ES_EINVAL / ES_ESTATE otherwise). */
es_status es_stash_and_switch(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                              const es_dtype *grad_dtypes, es_stash_mode mode, int32_t next_est, es_stream stream);

/* NEXT-1 incremental canonical fold (PAPER.md:599-606 overlaps
 * the gradient swap with the next EST's compute).  Every fold this rank runs
 * whose canonical sequence (R2: c+1, c+2, ... for chunk c) STARTS here -- at
 * G == 1 every chunk's whole sequence, for DIRECT / PEER the own shard's
 * chunks with EST c+1 local, for CHAIN / PEER_CHAIN a chain's first segment --
 * has a prefix of local ESTs c+1, c+2, ... (ascending, up to the wrap
 * N-1 -> 0, never the rank's last local EST, leaving the segment at least one
 * EST, and only if its q contributions outweigh the fp32 partial that replaces
 * them: q·b > 4 bytes, i.e. q >= 2 for fp32 and q >= 3 for bf16).  At the stash of a prefix EST its contribution is folded straight into
 * the running unrounded fp32 partial of that chunk (the first prefix EST opens
 * it); everything else of its gradient -- ranges peers or the exchange read,
 * chunks after the wrap -- is copied to the slot (COPY) or kept (BORROW).
 * es_allreduce then continues each such fold from its partial over the
 * remaining ESTs, so the end-of-step critical path reads fewer contributions
 * (G == 1: ~(N+3)/2 instead of N per element), with the same bits
 * (segmentability, R14).  Total bytes grow by the partials' round trips,
 * which the paper's overlap hides.
 * Requirements: cfg.options has ES_OPT_INCREMENTAL; every local EST of the
 * step calls this for the bucket, in ascending EST order (ES_ESTATE
 * otherwise; mixing with es_stash_grad for the same bucket and step is an
 * ES_ESTATE error).  mode: COPY (the unfolded part is copied) or BORROW (the
 * buffer is kept until es_allreduce completes).  A COPY-stashed EST whose
 * contribution was partly folded cannot be exported (es_export_context:
 * ES_ESTATE). */
es_status es_stash_fold_grads(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                              const es_dtype *grad_dtypes, es_stash_mode mode, es_stream stream);

/* ---- aggregation ---------------------------------------------------------- */

/* Collective over the G ranks: every rank calls it for the same bucket
 * sequence.  Requires every local EST to have stashed `bucket` since the
 * bucket's previous es_allreduce (ES_ESTATE otherwise).  Writes the
 * canonical average of all N ESTs' contributions (header comment) to
 * `out` (device, 16-byte aligned, numel elements of the bucket dtype) on
 * every rank.  `out` may alias a BORROWed gradient of this bucket; it may
 * not overlap the workspace.  Enqueued on `stream`; no host sync. */
es_status es_allreduce(es_handle h, int32_t bucket, void *out, es_stream stream);

/* Batched form of es_allreduce over n distinct buckets (host arrays), in the
 * given order; every rank must pass the same bucket sequence.  Independent
 * folds are merged into multi-segment launches (G == 1: one launch for all
 * buckets of a dtype).  Same argument rules and errors as es_allreduce,
 * checked for every entry before anything is enqueued. */
es_status es_allreduce_many(es_handle h, int32_t n, const int32_t *buckets, void *const *outs, es_stream stream);

/* ---- peer memory (ES_SCHED_PEER) -------------------------------------------- */

/* Opaque per-rank descriptor of this handle's workspace for peers: a CUDA
 * IPC handle of the workspace's allocation plus offset, process id and raw
 * address.  The caller all-gathers the G blobs with any collective it has
 * (e.g. torch.distributed.all_gather_object) and passes them, in rank order,
 * to es_peer_open, which maps every peer's workspace (cudaIpcOpenMemHandle
 * with lazy peer access; the raw address when the peer lives in the same
 * process, as with the loopback transport).  Required before the first
 * es_allreduce of a handle whose schedule is a peer one; ES_EUNSUPPORTED if
 * the workspace cannot be IPC-exported (e.g. a VMM / expandable-segments
 * allocation) or if more ranks share this process (loopback) than
 * CUDA_DEVICE_MAX_CONNECTIONS (default 8): their spinning barrier kernels
 * need a hardware queue each.  A peer that never arrives at a barrier makes
 * the kernel trap after 60 s (sticky ES_ECUDA), never hang the GPU. */
#define ES_PEER_BLOB_BYTES 128
es_status es_peer_blob(es_handle h, void *blob, size_t bytes);
es_status es_peer_open(es_handle h, const void *blobs, size_t bytes);

/* ---- zero-copy slots and elastic resume -------------- */

/* Device pointer of local EST `est`'s slot for `bucket` (bucket dtype,
 * numel elements, 256-byte aligned, inside the workspace).  A training loop
 * may bind EST est's gradient bucket there and stash with
 * ES_STASH_INPLACE: the stash then moves no bytes. */
es_status es_slot_ptr(es_handle h, int32_t est, int32_t bucket, void **ptr);

/* On-demand checkpoint of one EST's context ("EST
 * contexts" = RNG / BN state + the gradients already produced in this global
 * step), so that a job can be resumed on a different G / mapping mid-step
 * with bit-identical results (D1; synthetic Fig. 9).
 *   es_context_bytes: size of one exported context for this layout.
 *   es_export_context: writes local EST `est`'s context to host memory:
 *     header (layout hash of N, A, bucket numels/dtypes and state sizes --
 *     the persisted bucket indices of D1), which buckets are stashed, their
 *     contributions (from slot or borrowed buffer), and the saved (or, for the
 *     running EST, live) context buffers.  Synchronises `stream`.
 *   es_import_context: loads such a blob into local EST `est` of this handle
 *     (any G / mapping with the same N, A and layout; ES_ESTATE if the layout
 *     hash differs, ES_EINVAL if the blob is malformed).  Stashed buckets
 *     become stashed here (ordered on `stream`); state goes to the EST's
 *     slots (and to the live buffers if `est` is the running EST). */
es_status es_context_bytes(es_handle h, size_t *bytes);
es_status es_export_context(es_handle h, int32_t est, void *host_dst, size_t bytes, es_stream stream);
es_status es_import_context(es_handle h, int32_t est, const void *host_src, size_t bytes, es_stream stream);

/* ---- NEXT-4: a per-EST RNG consumer ---------------------------------------- */

/* Dropout of the running EST (Dropout "depends on the
 * random number generator (RNG) states"), driven on the device by the
 * 16-byte Philox record {seed u64, offset u64} registered as context buffer
 * `state_idx` -- the record es_switch_context swaps -- so the masks an EST
 * draws are the same whether it runs time-sliced or on a dedicated GPU, and
 * the call is CUDA-graph capturable.  Element i: Philox4x32-10 with key =
 * seed, counter = (i/4 lo, i/4 hi, offset lo, offset hi), word i % 4;
 * u = (w >> 8)*2^-24; kept iff u >= p; y = kept ? round(fl32(x*fl32(1/fl32(1-p)))) : +0.
 * One call consumes offset += 1 (advanced on the device).  x, y: device,
 * n elements of dtype, 16-byte aligned; mask: NULL or n bytes (1 = kept).
 * Calls on one handle must be stream-ordered.  ES_ESTATE if no EST is
 * running or no state is registered; ES_EINVAL for p outside [0, 1) or a
 * state_idx that is not a 16-byte buffer. */
es_status es_dropout(es_handle h, const void *x, void *y, uint8_t *mask, uint64_t n, es_dtype dtype, float p,
                     int32_t state_idx, es_stream stream);

/* ---- planner introspection (host-only, no CUDA) -------------------------- */

/* R1 chunk size C = A*ceil(ceil(L/N)/A) (A = 0 means 16). */
uint64_t es_chunk_elems(uint64_t L, int32_t N, uint32_t A);

/* Op-list export of the plan rank cfg->rank executes for `bucket`, so that
 * a host simulator can replay exactly what the GPU path does.  Each op is
 * ES_OP_FIELDS int64 values (layout below).  Writes up to cap_ops ops and
 * the total count to *n_ops; *sched_out gets the chosen es_sched (1/2; 0
 * when G == 1). */
#define ES_OP_FIELDS 10
enum {
  ES_OP_FOLD = 1,        /* [1]=lo [2]=hi [3]=e0 (-1: per-element rotation (c+1)%N) [4]=m (#ESTs)
                            [5]=in_kind (0 none / ES_BUF_PART / ES_BUF_PEER_PART) [6]=in_id
                                (PEER_PART: the producer rank)
                            [7]=out_kind (ES_BUF_PART: unscaled fp32 partial /
                                          ES_BUF_OUT / ES_BUF_RESULT: scaled, rounded) [8]=out_id
                                (PEER_CHAIN: byte offset of the own partial)
                            [9]=PEER_PART: byte offset in the producer's partials area       */
  ES_OP_SEND = 2,        /* [1]=lo [2]=hi [3]=peer [4]=buf_kind [5]=buf_id                      */
  ES_OP_RECV = 3,        /* same fields as SEND                                                 */
  ES_OP_GROUP_BEGIN = 4,
  ES_OP_GROUP_END = 5,
  ES_OP_BARRIER = 6,     /* PEER: all G ranks reach this point (device flags)                  */
  ES_OP_GATHER = 7       /* PEER: [1]=lo [2]=hi [3]=owner: out[lo,hi) <- owner's ES_BUF_RESULT  */
};
enum {
  ES_BUF_NONE = 0,
  ES_BUF_SRC = 1,        /* local EST buf_id's contribution (slot or borrowed), bucket dtype   */
  ES_BUF_STAGE = 2,      /* staging for remote EST buf_id's contribution, bucket dtype         */
  ES_BUF_PART = 3,       /* fp32 partial buffer buf_id                                         */
  ES_BUF_OUT = 4,        /* the caller's output, bucket dtype                                  */
  ES_BUF_RESULT = 5,     /* PEER: this rank's shard result area in its workspace, bucket dtype */
  ES_BUF_PEER_PART = 6   /* PEER_CHAIN: another rank's fp32 partial, read over NVLink          */
};
/* All [lo, hi) ranges are in bucket element coordinates. */
es_status es_plan_ops(const es_config *cfg, int32_t bucket, int64_t *ops, size_t cap_ops,
                      size_t *n_ops, int32_t *sched_out);

/* Host-only, like es_plan_ops: the NEXT-1 incremental prefixes of cfg->rank
 * for `bucket` (cfg->options must hold ES_OPT_INCREMENTAL, else *n_rows = 0).
 * Row i = rows[5i .. 5i+4] = {c, first, q, lo, hi}: at their stashes ESTs
 * first, first+1, ..., first+q-1 (first = (c+1) mod N) are folded into the
 * fp32 partial of bucket elements [lo, hi) of chunk c; es_allreduce
 * continues from it (see es_stash_fold_grads).  Rows ascend in c.  Same
 * two-call protocol as es_plan_ops (rows NULL: count only). */
es_status es_plan_incremental(const es_config *cfg, int32_t bucket, int64_t *rows, size_t cap_rows, size_t *n_rows);

/* ---- loopback transport (testing; see es_transport) ---------------------- */

es_status es_loopback_create(int32_t G, void **world);
es_status es_loopback_destroy(void *world);

/* ---- instrumentation ------------------------------------------------------ */

typedef enum {
  ES_KERNEL_STASH = 0, ES_KERNEL_FOLD = 1, ES_KERNEL_SWAP = 2, ES_KERNEL_DROPOUT = 3, ES_KERNEL_GATHER = 4,
  ES_KERNEL_BARRIER = 5, ES_KERNEL_KINDS = 6
} es_kernel_kind;

/* When enabled, every kernel launch of this handle is bracketed by CUDA
 * events on its own stream (event-record nodes when the stream is being
 * captured into a CUDA graph).  es_profile_query synchronises on those
 * events and returns, per kind since the last reset: launches, summed device
 * ms, and algorithmic bytes (reads + writes the method needs, DESIGN.md
 * "Kernels and their rooflines").  For captured launches the ms are those of
 * the graph's most recent replay and launches/bytes count the capture once.
 * Launch counts are kept even when timing is off. */
es_status es_profile_enable(es_handle h, int32_t on);
es_status es_profile_reset(es_handle h);
es_status es_profile_query(es_handle h, es_kernel_kind kind, uint64_t *launches, double *ms,
                           uint64_t *bytes);

/* Test hook (T4, launch-config invariance): force the
 * fold/stash grid size and block size; 0 restores the defaults.  Results
 * must not change. */
es_status es_set_launch_override(es_handle h, int32_t blocks, int32_t threads);

/* ---- errors --------------------------------------------------------------- */

const char *es_status_string(es_status s);
const char *es_last_error(void);
int32_t es_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ES_H */
