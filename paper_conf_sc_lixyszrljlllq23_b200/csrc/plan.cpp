// plan.cpp -- canonical plan: chunk table, shards, DIRECT / CHAIN exchange
// schedules, workspace layout.  See plan.h and DESIGN.md "Multi-GPU".
//
// Canonical order (readings R1-R3): chunk c of a bucket is
// folded over ESTs (c+1), (c+2), ..., (c+N) mod N -- the order a fixed-DoP
// N-worker ring all-reduce gives that chunk.
// Both schedules below realise exactly that order; they differ only in where
// the partial sums live and how many bytes cross NVLink.
#include "plan.h"
#include "kernels.h"

#include <algorithm>
#include <cstring>

namespace es {

uint64_t chunk_elems(uint64_t L, int32_t N, uint32_t A) {
  if (L == 0 || N <= 0 || A == 0) return 0;
  uint64_t per_rank = (L + (uint64_t)N - 1) / (uint64_t)N;
  return ((per_rank + A - 1) / A) * A;
}

namespace {

struct Seg {
  int32_t gpu, e0, m;  // GPU, first EST, number of consecutive ESTs (canonical order)
};

// Chunk c's canonical EST sequence (c+1 .. c+N mod N) cut into maximal runs
// of ESTs that live on the same GPU.  A left fold is segmentable: folding
// a run from the previous run's unrounded fp32 partial gives the same bits.
void chunk_segments(const Plan &p, int32_t c, std::vector<Seg> *out) {
  out->clear();
  for (int32_t j = 1; j <= p.N; ++j) {
    int32_t e = (int32_t)(((int64_t)c + j) % p.N);
    int32_t g = p.est_to_gpu[e];
    if (!out->empty() && out->back().gpu == g)
      out->back().m++;
    else
      out->push_back({g, e, 1});
  }
}

Op make_op(int64_t a0, int64_t a1 = 0, int64_t a2 = 0, int64_t a3 = 0, int64_t a4 = 0,
           int64_t a5 = 0, int64_t a6 = 0, int64_t a7 = 0, int64_t a8 = 0) {
  Op o;
  std::memset(&o, 0, sizeof(o));
  o.f[0] = a0; o.f[1] = a1; o.f[2] = a2; o.f[3] = a3; o.f[4] = a4;
  o.f[5] = a5; o.f[6] = a6; o.f[7] = a7; o.f[8] = a8;
  return o;
}

struct Range {
  int64_t lo, hi;
};

Range chunk_range(uint64_t L, uint64_t C, int32_t c) {
  int64_t lo = (int64_t)C * c, hi = std::min<int64_t>((int64_t)L, lo + (int64_t)C);
  if (lo > (int64_t)L) lo = (int64_t)L;
  return {lo, std::max(lo, hi)};
}

Range shard_range(uint64_t L, int32_t G, uint32_t A, int32_t h) {
  uint64_t S = chunk_elems(L, G, A);  // same rounding rule, G shards
  int64_t lo = std::min<int64_t>((int64_t)L, (int64_t)S * h);
  int64_t hi = std::min<int64_t>((int64_t)L, (int64_t)S * (h + 1));
  return {lo, hi};
}

// Bytes rank g receives per bucket under each schedule (used by AUTO).
uint64_t direct_recv_bytes(const Plan &p, const BucketPlan &b, int32_t g) {
  int32_t ng = 0;
  for (int32_t e = 0; e < p.N; ++e) ng += p.est_to_gpu[e] == g;
  Range s = shard_range(b.L, p.G, p.A, g);
  uint64_t own = (uint64_t)(s.hi - s.lo);
  return (uint64_t)(p.N - ng) * own * b.esize + (b.L - own) * b.esize;
}

uint64_t chain_recv_bytes(const Plan &p, const BucketPlan &b, int32_t g) {
  uint64_t bytes = 0;
  std::vector<Seg> segs;
  for (int32_t c = 0; c < p.N; ++c) {
    Range r = chunk_range(b.L, b.C, c);
    if (r.hi <= r.lo) continue;
    chunk_segments(p, c, &segs);
    for (size_t s = 1; s < segs.size(); ++s)
      if (segs[s].gpu == g) bytes += (uint64_t)(r.hi - r.lo) * 4;  // fp32 partial in
    if (p.est_to_gpu[c] != g) bytes += (uint64_t)(r.hi - r.lo) * b.esize;  // gather in
  }
  return bytes;
}

void plan_single(const Plan &p, BucketPlan *b) {
  b->sched = 0;
  if (b->L == 0) return;
  b->ops.push_back(make_op(ES_OP_FOLD, 0, (int64_t)b->L, -1, p.N, ES_BUF_NONE, 0, ES_BUF_OUT, 0));
}

void plan_direct(const Plan &p, BucketPlan *b) {
  const int32_t g = p.rank;
  b->sched = ES_SCHED_DIRECT;
  if (b->L == 0) return;
  Range own = shard_range(b->L, p.G, p.A, g);
  b->shard_lo = own.lo;
  b->shard_hi = own.hi;
  const bool have = own.hi > own.lo;
  // Staging: one slot per remote EST, holding its contribution to S_g.
  b->stage_index.assign(p.N, -1);
  int32_t ns = 0;
  if (have)
    for (int32_t e = 0; e < p.N; ++e)
      if (p.est_to_gpu[e] != g) b->stage_index[e] = ns++;
  b->stage_stride = align256((uint64_t)(own.hi - own.lo) * b->esize);
  b->stage_bytes = b->stage_stride * (uint64_t)ns;

  // 1. exchange: send my ESTs' slices of every peer's shard, receive the
  //    remote ESTs' slices of mine.  Per (src, dst) pair both sides post in
  //    ascending EST order, so point-to-point matching is exact.
  b->ops.push_back(make_op(ES_OP_GROUP_BEGIN));
  for (int32_t k : p.local_ests)
    for (int32_t h = 0; h < p.G; ++h) {
      if (h == g) continue;
      Range s = shard_range(b->L, p.G, p.A, h);
      if (s.hi > s.lo) b->ops.push_back(make_op(ES_OP_SEND, s.lo, s.hi, h, ES_BUF_SRC, k));
    }
  if (have)
    for (int32_t e = 0; e < p.N; ++e)
      if (p.est_to_gpu[e] != g)
        b->ops.push_back(make_op(ES_OP_RECV, own.lo, own.hi, p.est_to_gpu[e], ES_BUF_STAGE, e));
  b->ops.push_back(make_op(ES_OP_GROUP_END));
  // 2. canonical fold of all N contributions over the own shard.
  if (have) b->ops.push_back(make_op(ES_OP_FOLD, own.lo, own.hi, -1, p.N, ES_BUF_NONE, 0, ES_BUF_OUT, 0));
  // 3. all-gather of the shards (pure copies, exact sizes, no padding).
  b->ops.push_back(make_op(ES_OP_GROUP_BEGIN));
  for (int32_t h = 0; h < p.G; ++h)
    if (h != g && have) b->ops.push_back(make_op(ES_OP_SEND, own.lo, own.hi, h, ES_BUF_OUT, 0));
  for (int32_t h = 0; h < p.G; ++h) {
    if (h == g) continue;
    Range s = shard_range(b->L, p.G, p.A, h);
    if (s.hi > s.lo) b->ops.push_back(make_op(ES_OP_RECV, s.lo, s.hi, h, ES_BUF_OUT, 0));
  }
  b->ops.push_back(make_op(ES_OP_GROUP_END));
}

// PEER (fused pull over peer memory): barrier (every rank's slots hold
// this step's contributions) -> fold of the own shard reading remote
// contributions from the owners' slots, result into the own RESULT area ->
// barrier (every shard result is ready; every slot has been read) -> gather
// of every shard from its owner's RESULT area into out.
void plan_peer(const Plan &p, BucketPlan *b) {
  const int32_t g = p.rank;
  b->sched = ES_SCHED_PEER;
  if (b->L == 0) return;
  Range own = shard_range(b->L, p.G, p.A, g);
  b->shard_lo = own.lo;
  b->shard_hi = own.hi;
  b->ops.push_back(make_op(ES_OP_BARRIER, 0));
  if (own.hi > own.lo)
    b->ops.push_back(make_op(ES_OP_FOLD, own.lo, own.hi, -1, p.N, ES_BUF_NONE, 0, ES_BUF_RESULT, 0));
  b->ops.push_back(make_op(ES_OP_BARRIER, 1));
  for (int32_t h = 0; h < p.G; ++h) {
    Range s = shard_range(b->L, p.G, p.A, h);
    if (s.hi > s.lo) b->ops.push_back(make_op(ES_OP_GATHER, s.lo, s.hi, h));
  }
}

void plan_chain(const Plan &p, BucketPlan *b) {
  const int32_t g = p.rank;
  b->sched = ES_SCHED_CHAIN;
  if (b->L == 0) return;
  const int32_t N = p.N;
  std::vector<std::vector<Seg>> segs(N);
  std::vector<Range> rng(N);
  int32_t R = 0;
  for (int32_t c = 0; c < N; ++c) {
    rng[c] = chunk_range(b->L, b->C, c);
    if (rng[c].hi <= rng[c].lo) continue;
    chunk_segments(p, c, &segs[c]);
    R = std::max<int32_t>(R, (int32_t)segs[c].size());
  }
  // Partial buffers: in_id[c][r] (incoming partial of segment r, r > 0) and
  // out_id[c][r] (outgoing partial of segment r, r < last), for segments on g.
  std::vector<std::vector<int32_t>> in_id(N), out_id(N);
  uint64_t off = 0;
  auto new_part = [&](const Range &r) {
    b->parts.push_back({r.lo, r.hi, off});
    off += align256((uint64_t)(r.hi - r.lo) * 4);
    return (int32_t)b->parts.size() - 1;
  };
  for (int32_t r = 0; r < R; ++r)
    for (int32_t c = 0; c < N; ++c) {
      int32_t m = (int32_t)segs[c].size();
      if (r == 0) { in_id[c].assign(m, -1); out_id[c].assign(m, -1); }
      if (r >= m || segs[c][r].gpu != g) continue;
      if (r > 0) in_id[c][r] = new_part(rng[c]);
      if (r < m - 1) out_id[c][r] = new_part(rng[c]);
    }
  b->part_bytes = off;

  for (int32_t r = 0; r < R; ++r) {
    for (int32_t c = 0; c < N; ++c) {
      int32_t m = (int32_t)segs[c].size();
      if (r >= m || segs[c][r].gpu != g) continue;
      const Seg &s = segs[c][r];
      b->ops.push_back(make_op(ES_OP_FOLD, rng[c].lo, rng[c].hi, s.e0, s.m,
                               r > 0 ? ES_BUF_PART : ES_BUF_NONE, r > 0 ? in_id[c][r] : 0,
                               r == m - 1 ? ES_BUF_OUT : ES_BUF_PART, r == m - 1 ? 0 : out_id[c][r]));
    }
    if (r + 1 >= R) break;
    std::vector<Op> xs;
    for (int32_t c = 0; c < N; ++c) {
      int32_t m = (int32_t)segs[c].size();
      if (r < m - 1 && segs[c][r].gpu == g)
        xs.push_back(make_op(ES_OP_SEND, rng[c].lo, rng[c].hi, segs[c][r + 1].gpu, ES_BUF_PART,
                             out_id[c][r]));
    }
    for (int32_t c = 0; c < N; ++c) {
      int32_t m = (int32_t)segs[c].size();
      if (r + 1 < m && segs[c][r + 1].gpu == g)
        xs.push_back(make_op(ES_OP_RECV, rng[c].lo, rng[c].hi, segs[c][r].gpu, ES_BUF_PART,
                             in_id[c][r + 1]));
    }
    if (!xs.empty()) {
      b->ops.push_back(make_op(ES_OP_GROUP_BEGIN));
      b->ops.insert(b->ops.end(), xs.begin(), xs.end());
      b->ops.push_back(make_op(ES_OP_GROUP_END));
    }
    b->op_round.resize(b->ops.size(), r);
  }
  b->op_round.resize(b->ops.size(), R > 0 ? R - 1 : 0);   // last round's folds (the loop broke early)
  // All-gather: chunk c is finished (scaled, rounded) on the GPU of EST c,
  // the last EST of its sequence; it sends the chunk to every peer.
  b->ops.push_back(make_op(ES_OP_GROUP_BEGIN));
  for (int32_t c = 0; c < N; ++c) {
    if (rng[c].hi <= rng[c].lo) continue;
    int32_t owner = p.est_to_gpu[c];
    if (owner == g) {
      for (int32_t h = 0; h < p.G; ++h)
        if (h != g) b->ops.push_back(make_op(ES_OP_SEND, rng[c].lo, rng[c].hi, h, ES_BUF_OUT, 0));
    } else {
      b->ops.push_back(make_op(ES_OP_RECV, rng[c].lo, rng[c].hi, owner, ES_BUF_OUT, 0));
    }
  }
  b->ops.push_back(make_op(ES_OP_GROUP_END));
  b->op_round.resize(b->ops.size(), -1);
}

// ---- PEER_CHAIN ----------------------------------------------------------------
// The CHAIN schedule without a transport: the GPU of segment r of chunk c
// reads the incoming unrounded fp32 partial directly out of the producer's
// workspace over NVLink (part_in = a peer pointer) inside its fold kernel, so
// the partial's transfer and the local fold are one kernel.  The op list keeps
// a BARRIER between rounds; the default executor replaces those inner barriers
// by per-tile flags (k_fold_pipe, tile flags at pipe_flag_base) and keeps only
// the first and the last; ES_OPT_PEER_ROUNDS executes them as written.  Chunk
// c ends in the RESULT area of the GPU of EST c and is gathered from there.

struct ChainShape {
  std::vector<std::vector<Seg>> segs;
  std::vector<Range> rng;
  int32_t R = 0;
};

ChainShape chain_shape(const Plan &p, const BucketPlan &b) {
  ChainShape sh;
  sh.segs.resize(p.N);
  sh.rng.resize(p.N);
  for (int32_t c = 0; c < p.N; ++c) {
    sh.rng[c] = chunk_range(b.L, b.C, c);
    if (sh.rng[c].hi <= sh.rng[c].lo) continue;
    chunk_segments(p, c, &sh.segs[c]);
    sh.R = std::max<int32_t>(sh.R, (int32_t)sh.segs[c].size());
  }
  return sh;
}

// Byte offsets (inside the uniform peer partials area) of rank h's outgoing
// partials, off[c][r] (-1: none), allocated in (round, chunk) order; returns
// the bytes rank h needs.
uint64_t chain_out_parts(const ChainShape &sh, int32_t h, std::vector<std::vector<int64_t>> *off) {
  const int32_t N = (int32_t)sh.segs.size();
  off->assign(N, {});
  for (int32_t c = 0; c < N; ++c) (*off)[c].assign(sh.segs[c].size(), -1);
  uint64_t o = 0;
  for (int32_t r = 0; r < sh.R; ++r)
    for (int32_t c = 0; c < N; ++c) {
      const int32_t m = (int32_t)sh.segs[c].size();
      if (r >= m - 1 || sh.segs[c][r].gpu != h) continue;
      (*off)[c][r] = (int64_t)o;
      o += align256((uint64_t)(sh.rng[c].hi - sh.rng[c].lo) * 4);
    }
  return o;
}

void plan_peer_chain(const Plan &p, BucketPlan *b) {
  const int32_t g = p.rank;
  b->sched = ES_SCHED_PEER_CHAIN;
  if (b->L == 0) return;
  const ChainShape sh = chain_shape(p, *b);
  std::vector<std::vector<std::vector<int64_t>>> offs(p.G);
  for (int32_t h = 0; h < p.G; ++h) b->peer_part_bytes = std::max(b->peer_part_bytes, chain_out_parts(sh, h, &offs[h]));
  b->part_bytes = 0;
  b->chain_rounds = sh.R;
  b->tiles_per_chunk = (b->C + kPipeTile - 1) / kPipeTile;
  b->ops.push_back(make_op(ES_OP_BARRIER, 0));
  for (int32_t r = 0; r < sh.R; ++r) {
    for (int32_t c = 0; c < p.N; ++c) {
      const int32_t m = (int32_t)sh.segs[c].size();
      if (r >= m || sh.segs[c][r].gpu != g) continue;
      const Seg &s = sh.segs[c][r];
      Op o = make_op(ES_OP_FOLD, sh.rng[c].lo, sh.rng[c].hi, s.e0, s.m, ES_BUF_NONE, 0,
                     r == m - 1 ? ES_BUF_RESULT : ES_BUF_PART, 0);
      if (r > 0) {                       // incoming partial: the producer's buffer, over NVLink
        const int32_t prod = sh.segs[c][r - 1].gpu;
        o.f[5] = ES_BUF_PEER_PART;
        o.f[6] = prod;
        o.f[9] = offs[prod][c][r - 1];
      }
      if (r < m - 1) o.f[8] = offs[g][c][r];   // own outgoing partial (byte offset)
      b->ops.push_back(o);
    }
    b->ops.push_back(make_op(ES_OP_BARRIER, r + 1));
  }
  for (int32_t c = 0; c < p.N; ++c)
    if (sh.rng[c].hi > sh.rng[c].lo)
      b->ops.push_back(make_op(ES_OP_GATHER, sh.rng[c].lo, sh.rng[c].hi, p.est_to_gpu[c]));
}

// NEXT-1 (PAPER.md:599-606 overlaps the gradient swap with the
// next EST's compute): which ESTs of which chunks this rank can fold into a
// running fp32 partial at their stashes, before any exchange.  A left fold is
// segmentable (R14), so the partial of the first q ESTs of a sequence that
// starts here, continued by the end fold over the rest, gives the same bits.
// Local ESTs stash in ascending order, so the prefix stops at the wrap
// N-1 -> 0; it never takes the last local EST (nothing is left to overlap
// with after its stash, and the end fold reads it straight from its stash)
// and leaves the segment's end fold at least one source.  A prefix is taken only if its q
// contributions outweigh the fp32 partial that replaces them in the end fold (q·b > 4 bytes).
void plan_incremental(const Plan &p, BucketPlan *b) {
  b->inc.clear();
  b->inc_q.assign(p.N, 0);
  if (b->L == 0 || p.local_ests.empty()) return;
  const int32_t g = p.rank, last_local = p.local_ests.back();
  const bool shard = b->sched == ES_SCHED_DIRECT || b->sched == ES_SCHED_PEER;
  std::vector<Seg> segs;
  for (int32_t c = 0; c < p.N; ++c) {
    Range r = chunk_range(b->L, b->C, c);
    const int32_t first = (int32_t)(((int64_t)c + 1) % p.N);
    if (p.est_to_gpu[first] != g) continue;   // the sequence does not start here
    if (shard) {
      r.lo = std::max<int64_t>(r.lo, b->shard_lo);
      r.hi = std::min<int64_t>(r.hi, b->shard_hi);
    }
    if (r.hi <= r.lo) continue;
    int32_t seg_len = p.N;                    // G == 1, DIRECT, PEER: the whole sequence folds here
    if (b->sched == ES_SCHED_CHAIN || b->sched == ES_SCHED_PEER_CHAIN) {
      chunk_segments(p, c, &segs);
      seg_len = segs[0].m;                    // the chain's first segment (on this rank)
    }
    int32_t q = 0;
    while (q < seg_len - 1) {
      const int32_t e = first + q;
      if (e >= p.N || p.est_to_gpu[e] != g || e == last_local) break;
      ++q;
    }
    // worth it only if the end fold then reads fewer bytes: q contributions (q*b) become one
    // fp32 partial (4 B) -- fp32 needs q >= 2, bf16 q >= 3
    if ((uint64_t)q * b->esize <= 4) continue;
    b->inc_q[c] = q;
    b->inc.push_back({c, first, q, r.lo, r.hi});
  }
}

bool fail(std::string *err, const char *msg) {
  if (err) *err = msg;
  return false;
}

bool validate(const es_config *cfg, std::string *err, bool need_comm) {
  if (!cfg) return fail(err, "config is NULL");
  if (cfg->N < 1 || cfg->N > 1024) return fail(err, "N must be in [1, 1024]");
  if (cfg->G < 1 || cfg->G > 64) return fail(err, "G must be in [1, 64]");
  if (cfg->G > cfg->N) return fail(err, "G must be <= N (every GPU owns >= 1 EST, R10)");
  if (cfg->rank < 0 || cfg->rank >= cfg->G) return fail(err, "rank must be in [0, G)");
  if (!cfg->est_to_gpu) return fail(err, "est_to_gpu is NULL");
  std::vector<int32_t> cnt(cfg->G, 0);
  for (int32_t e = 0; e < cfg->N; ++e) {
    int32_t g = cfg->est_to_gpu[e];
    if (g < 0 || g >= cfg->G) return fail(err, "est_to_gpu value out of [0, G)");
    cnt[g]++;
  }
  for (int32_t g = 0; g < cfg->G; ++g)
    if (cnt[g] == 0) return fail(err, "every GPU must own at least one EST (R10)");
  if (cfg->n_buckets < 1 || cfg->n_buckets > 4096) return fail(err, "n_buckets must be in [1, 4096]");
  if (!cfg->buckets) return fail(err, "buckets is NULL");
  for (int32_t b = 0; b < cfg->n_buckets; ++b) {
    if (cfg->buckets[b].numel >= (1ull << 31)) return fail(err, "bucket numel must be < 2^31");
    if (cfg->buckets[b].dtype != ES_F32 && cfg->buckets[b].dtype != ES_BF16)
      return fail(err, "bucket dtype must be ES_F32 or ES_BF16");
  }
  uint32_t A = cfg->chunk_align ? cfg->chunk_align : 16;
  if (A % 8 != 0 || A > (1u << 20)) return fail(err, "chunk_align must be a multiple of 8 and <= 2^20");
  if (cfg->n_state < 0 || cfg->n_state > 4096) return fail(err, "n_state must be in [0, 4096]");
  if (cfg->n_state > 0 && !cfg->state_nbytes) return fail(err, "state_nbytes is NULL");
  for (int32_t i = 0; i < cfg->n_state; ++i)
    if (cfg->state_nbytes[i] == 0 || cfg->state_nbytes[i] > (1ull << 31))
      return fail(err, "state_nbytes must be in [1, 2^31]");
  if (cfg->sched != ES_SCHED_AUTO && cfg->sched != ES_SCHED_DIRECT && cfg->sched != ES_SCHED_CHAIN &&
      cfg->sched != ES_SCHED_PEER && cfg->sched != ES_SCHED_PEER_CHAIN && cfg->sched != ES_SCHED_PEER_AUTO)
    return fail(err, "bad sched");
  if (cfg->compat & ~(uint32_t)(ES_COMPAT_PREDIV | ES_COMPAT_PREMUL | ES_COMPAT_BF16_HOP))
    return fail(err, "unknown compat bits");
  if ((cfg->compat & ES_COMPAT_PREDIV) && (cfg->compat & ES_COMPAT_PREMUL))
    return fail(err, "compat PREDIV and PREMUL are exclusive");
  if (cfg->options & ~(uint32_t)(ES_OPT_INCREMENTAL | ES_OPT_PEER_ROUNDS | ES_OPT_STASH_BACKGROUND | ES_OPT_PEER_PUSH))
    return fail(err, "unknown option bits");
  const bool peer_sched = cfg->sched == ES_SCHED_PEER || cfg->sched == ES_SCHED_PEER_CHAIN ||
                          cfg->sched == ES_SCHED_PEER_AUTO;
  if (cfg->G > 1 && need_comm && !peer_sched) {
    if (cfg->transport != ES_TRANSPORT_NCCL && cfg->transport != ES_TRANSPORT_LOOPBACK)
      return fail(err, "G > 1 needs transport NCCL or LOOPBACK");
    if (!cfg->comm) return fail(err, "G > 1 needs comm");
  } else if (cfg->transport != ES_TRANSPORT_NONE && cfg->transport != ES_TRANSPORT_NCCL &&
             cfg->transport != ES_TRANSPORT_LOOPBACK) {
    return fail(err, "bad transport");
  }
  return true;
}

}  // namespace

es_status build_plan(const es_config *cfg, Plan *p, std::string *err, bool need_comm) {
  if (!validate(cfg, err, need_comm)) return ES_EINVAL;
  *p = Plan();
  p->N = cfg->N;
  p->G = cfg->G;
  p->rank = cfg->rank;
  p->A = cfg->chunk_align ? cfg->chunk_align : 16;
  p->est_to_gpu.assign(cfg->est_to_gpu, cfg->est_to_gpu + cfg->N);
  p->local_index.assign(cfg->N, -1);
  for (int32_t e = 0; e < cfg->N; ++e)
    if (p->est_to_gpu[e] == p->rank) {
      p->local_index[e] = (int32_t)p->local_ests.size();
      p->local_ests.push_back(e);
    }
  p->buckets.assign(cfg->buckets, cfg->buckets + cfg->n_buckets);
  if (cfg->n_state > 0) p->state_nbytes.assign(cfg->state_nbytes, cfg->state_nbytes + cfg->n_state);
  p->transport = cfg->G > 1 ? cfg->transport : ES_TRANSPORT_NONE;
  p->comm = cfg->G > 1 ? cfg->comm : nullptr;
  p->sched_req = cfg->sched;
  p->compat = cfg->compat;
  p->options = cfg->options;

  p->bp.resize(cfg->n_buckets);
  uint64_t max_stage = 0, max_parts = 0, sum_parts = 0, sum_peer_parts = 0, sum_pipe_flags = 0;
  // CHAIN over a transport, tile-pipelined (chain_pipelined): all chain buckets of one
  // es_allreduce_many are in flight together, so each owns its partial buffers
  const bool chain_pipe = cfg->G > 1 && !(cfg->options & ES_OPT_PEER_ROUNDS);
  for (int32_t bi = 0; bi < cfg->n_buckets; ++bi) {
    BucketPlan &b = p->bp[bi];
    b.L = p->buckets[bi].numel;
    b.dtype = p->buckets[bi].dtype;
    b.esize = dtype_size(b.dtype);
    b.C = chunk_elems(b.L, p->N, p->A);
    if (p->G == 1) {
      plan_single(*p, &b);
    } else {
      es_sched s = p->sched_req;
      if (s == ES_SCHED_AUTO || s == ES_SCHED_PEER_AUTO) {
        uint64_t d = 0, ch = 0;
        for (int32_t g = 0; g < p->G; ++g) {
          d = std::max(d, direct_recv_bytes(*p, b, g));
          ch = std::max(ch, chain_recv_bytes(*p, b, g));
        }
        const bool chain = ch < d;
        if (s == ES_SCHED_AUTO) s = chain ? ES_SCHED_CHAIN : ES_SCHED_DIRECT;
        else s = chain ? ES_SCHED_PEER_CHAIN : ES_SCHED_PEER;
      }
      if (s == ES_SCHED_CHAIN) plan_chain(*p, &b);
      else if (s == ES_SCHED_PEER) plan_peer(*p, &b);
      else if (s == ES_SCHED_PEER_CHAIN) plan_peer_chain(*p, &b);
      else plan_direct(*p, &b);
    }
    if (p->options & ES_OPT_INCREMENTAL) plan_incremental(*p, &b);
    max_stage = std::max(max_stage, b.stage_bytes);
    max_parts = std::max(max_parts, b.part_bytes);
    b.part_base = chain_pipe ? sum_parts : 0;
    sum_parts += chain_pipe ? align256(b.part_bytes) : 0;
    b.peer_part_base = sum_peer_parts;   // buckets of one batched call run their rounds together
    sum_peer_parts += align256(b.peer_part_bytes);
    if (b.sched == ES_SCHED_PEER_CHAIN) {
      b.pipe_flag_base = sum_pipe_flags;
      sum_pipe_flags += (uint64_t)p->N * (uint64_t)b.chain_rounds * b.tiles_per_chunk;
    }
  }

  // Workspace layout.
  uint64_t off = 0;
  p->slot_off.resize(cfg->n_buckets);
  for (int32_t bi = 0; bi < cfg->n_buckets; ++bi) {
    p->slot_off[bi] = off;
    off += align256(p->bp[bi].L * p->bp[bi].esize);
  }
  p->slot_block = off;
  // PEER: the regions peers address (flags, shard results, gradient slots)
  // come first, at offsets that depend only on the layout -- identical on
  // every rank whatever its number of local ESTs.
  p->peer = p->G > 1 && (p->sched_req == ES_SCHED_PEER || p->sched_req == ES_SCHED_PEER_CHAIN ||
                          p->sched_req == ES_SCHED_PEER_AUTO);
  uint64_t head = 0;
  if (p->peer) {
    p->flags_off = 0;
    p->result_off = align256(kPeerFlagWords * 8);   // G flags + the epoch counter
    head = p->result_off + p->slot_block;   // one bucket-layout block: shard results at bucket offsets
    p->peer_parts_off = head;               // PEER_CHAIN partials: per bucket, max over ranks
    head += align256(sum_peer_parts);
    p->pipe_flags_off = head;               // PEER_CHAIN tile flags (k_fold_pipe)
    p->pipe_flag_words = sum_pipe_flags;
    head += align256(sum_pipe_flags * 8);
  }
  p->grad_off = head;
  uint64_t total = head + p->slot_block * p->local_ests.size();
  off = 0;
  p->state_off.resize(p->state_nbytes.size());
  for (size_t i = 0; i < p->state_nbytes.size(); ++i) {
    p->state_off[i] = off;
    off += align256(p->state_nbytes[i]);
  }
  p->state_block = off;
  p->state_area_off = total;
  total += p->state_block * p->local_ests.size();
  p->table_off = total;
  total += align256(p->state_nbytes.size() * 32);
  p->scratch_off = total;
  total += 256;
  p->stage_off = total;
  total += max_stage;
  p->parts_off = total;
  total += chain_pipe ? sum_parts : max_parts;
  if (p->options & ES_OPT_INCREMENTAL) {
    p->inc_off = align256(total);
    uint64_t o = 0;
    p->inc_bucket_off.resize(p->bp.size());
    for (size_t bi = 0; bi < p->bp.size(); ++bi) {
      p->inc_bucket_off[bi] = o;
      o += align256(p->bp[bi].L * 4);
    }
    total = p->inc_off + o;
  }
  p->owner_index.assign(p->N, 0);
  {
    std::vector<int32_t> cnt(p->G, 0);
    for (int32_t e = 0; e < p->N; ++e) p->owner_index[e] = cnt[p->est_to_gpu[e]]++;
  }
  p->total = align256(total);
  return ES_OK;
}

}  // namespace es
