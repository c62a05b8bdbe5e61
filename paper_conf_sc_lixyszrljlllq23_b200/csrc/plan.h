// plan.h -- host planner of libes ("canonical plan").
//
// Everything the GPU path does for a bucket is decided here, once, at
// es_init, from (N, G, rank, EST->GPU mapping, bucket layout, A) only:
// the R1 chunk table, the element shards, the exchange schedule and the
// exact op list each rank executes.  The plan is never rebuilt while the
// handle lives -- the D1 rule "reconstruction of the communication channel
// is disabled".
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "../../include/es.h"

namespace es {

struct Op {
  int64_t f[ES_OP_FIELDS];
};

// fp32 partial buffer: bucket element range [lo, hi) at byte offset `off`
// of the partials area.
struct Part {
  int64_t lo, hi;
  uint64_t off;
};

// NEXT-1 (incremental fold): a chunk whose canonical sequence starts on this
// rank (the first segment of a chain, or the local run opening a DIRECT/PEER
// shard fold) folds its first q ESTs into fp32 partials at their stashes.
// [lo, hi): the elements this rank folds for the chunk (chunk, or chunk and
// shard); first = (c+1) mod N.  q >= 1 only; q ends before the wrap N-1 -> 0
// (ESTs run in ascending order), never takes this rank's last local EST (its
// contribution joins the end fold straight from its stash) and leaves at least
// one source of the segment to the end fold; only prefixes with q·b > 4 (they must save more
// end-fold reads than the 4-byte partial costs) are kept.
struct IncChunk {
  int32_t c, first, q;
  int64_t lo, hi;
};

struct BucketPlan {
  uint64_t L = 0;
  es_dtype dtype = ES_F32;
  uint32_t esize = 4;            // bytes per element of the bucket dtype
  uint64_t C = 0;                // R1 chunk size
  int32_t sched = 0;             // 0: G == 1, ES_SCHED_DIRECT, ES_SCHED_CHAIN
  int64_t shard_lo = 0, shard_hi = 0;   // DIRECT: this rank's shard
  std::vector<int32_t> stage_index;     // [N]: staging slot of remote EST, -1 if local/unused
  uint64_t stage_stride = 0;            // bytes per staging slot
  uint64_t stage_bytes = 0;
  std::vector<Part> parts;
  uint64_t part_bytes = 0;
  uint64_t part_base = 0;               // CHAIN: this bucket's base in the partials area (0 when the
                                        //   round executor reuses one area bucket after bucket)
  uint64_t peer_part_bytes = 0;         // PEER_CHAIN: max over ranks of their outgoing partials
  uint64_t peer_part_base = 0;          // PEER_CHAIN: this bucket's base in the peer partials area
  int32_t chain_rounds = 0;             // PEER_CHAIN: R, the most segments of any chunk (all ranks)
  uint64_t tiles_per_chunk = 0;         // PEER_CHAIN: ceil(C / kPipeTile)
  uint64_t pipe_flag_base = 0;          // PEER_CHAIN: first tile flag (u64 words) of this bucket;
                                        //   chunk c, round r, tile t at base + (c*R + r)*tiles_per_chunk + t
  std::vector<Op> ops;
  std::vector<int32_t> op_round;        // CHAIN: [ops] round of a fold / of the transfer group after
                                        //   that round's folds; -1: the final all-gather group
  std::vector<IncChunk> inc;            // NEXT-1 (ES_OPT_INCREMENTAL): chunks with q >= 1, ascending c
  std::vector<int32_t> inc_q;           // NEXT-1: [N] q of chunk c on this rank (0: none)
};

struct Plan {
  int32_t N = 0, G = 0, rank = 0;
  uint32_t A = 16;
  std::vector<int32_t> est_to_gpu;
  std::vector<int32_t> local_ests;      // ascending
  std::vector<int32_t> local_index;     // [N] -> index into local_ests, -1 if remote
  std::vector<es_bucket_desc> buckets;
  std::vector<uint64_t> state_nbytes;
  es_transport transport = ES_TRANSPORT_NONE;
  void *comm = nullptr;
  es_sched sched_req = ES_SCHED_AUTO;
  uint32_t compat = 0;                  // NEXT-3 variant bits
  uint32_t options = 0;                 // ES_OPT_* bits
  uint64_t inc_off = 0;                 // NEXT-1: fp32 partials, bucket-major (inc_block bytes)
  std::vector<uint64_t> inc_bucket_off; // [n_buckets]
  std::vector<BucketPlan> bp;

  // Workspace layout (byte offsets from the workspace base, 256-aligned).
  std::vector<uint64_t> slot_off;       // [n_buckets]: offset inside one EST's gradient block
  uint64_t slot_block = 0;              // bytes of one EST's gradient block
  uint64_t grad_off = 0;                // n_local gradient blocks
  std::vector<uint64_t> state_off;      // [n_state]: offset inside one EST's state block
  uint64_t state_block = 0;
  uint64_t state_area_off = 0;          // n_local state blocks
  uint64_t table_off = 0;               // swap table (n_state entries)
  uint64_t scratch_off = 0;             // 256 B of zeroed scratch (dropout grid counter)
  uint64_t stage_off = 0;               // exchange staging (max over buckets)
  uint64_t parts_off = 0;               // chain partials: max over buckets (round executor), or the
                                        //   sum (tile-pipelined: every bucket of a call in flight at once)
  uint64_t flags_off = 0;               // PEER: G barrier flags (u64) written by peers + epoch counter
  uint64_t result_off = 0;              // PEER: per-bucket shard results (slot-block layout)
  uint64_t peer_parts_off = 0;          // PEER_CHAIN: partials read by the next GPU (uniform offset)
  uint64_t pipe_flags_off = 0;          // PEER_CHAIN: per-tile publish flags (uniform offset)
  uint64_t pipe_flag_words = 0;
  bool peer = false;                    // some bucket uses ES_SCHED_PEER
  std::vector<int32_t> owner_index;     // [N]: EST's index among its owner's local ESTs
  uint64_t total = 0;
};

inline uint64_t align256(uint64_t x) { return (x + 255) & ~uint64_t(255); }
inline uint32_t dtype_size(es_dtype d) { return d == ES_BF16 ? 2u : 4u; }

// R1: C = A * ceil(ceil(L / N) / A).
uint64_t chunk_elems(uint64_t L, int32_t N, uint32_t A);

// Validates cfg and builds the full plan for cfg->rank.  On failure returns
// ES_EINVAL and sets *err.
// need_comm == false (host-only queries) skips the transport/comm checks.
es_status build_plan(const es_config *cfg, Plan *plan, std::string *err, bool need_comm = true);

}  // namespace es
