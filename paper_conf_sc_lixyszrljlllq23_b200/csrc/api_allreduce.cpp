// api_allreduce.cpp -- C ABI: es_allreduce(_many), the executor that walks the
// planner's op list (plan.cpp) launching multi-segment folds and transport
// groups, and the phase-merged ES_SCHED_PEER executor.
#include <unistd.h>

#include "handle.h"

extern "C" {

// ---- aggregation --------------------------------------------------------------------

namespace {
es_status finish_allreduce(es_handle h, int32_t n, const int32_t *buckets, cudaStream_t cs, unsigned long long cap);

// NEXT-1 end of step.  A planned fold over [lo, hi) that starts its sequence
// fresh -- rot (every chunk's whole canonical sequence: G == 1, DIRECT, PEER)
// or a chain's first segment (ESTs e0, e0+1, ..., m of them) -- is cut into
// per-chunk pieces; where plan_incremental folded the first q ESTs of chunk c
// into the fp32 partial at their stashes, the piece continues from that
// partial over the remaining ESTs of the sequence (segmentability, R14).
// Chunks without a partial stay rot pieces (merged when adjacent).
struct Piece {
  int64_t lo, hi;
  bool rot;
  int32_t e0, m;
  bool part;
};
void inc_pieces(const es::Plan &p, const es::BucketPlan &b, bool inc, int64_t lo, int64_t hi, int64_t e0, int32_t m,
                std::vector<Piece> *out) {
  out->clear();
  if (!inc) {
    out->push_back({lo, hi, e0 < 0, (int32_t)e0, m, false});
    return;
  }
  const int64_t C = (int64_t)b.C;
  for (int64_t a = lo; a < hi;) {
    const int32_t c = (int32_t)(a / C);
    const int64_t z = std::min<int64_t>(hi, (int64_t)(c + 1) * C);
    const int32_t q = b.inc_q[c];
    if (q == 0) {
      if (e0 < 0 && !out->empty() && out->back().rot && out->back().hi == a) out->back().hi = z;
      else out->push_back({a, z, e0 < 0, (int32_t)e0, m, false});
    } else if (e0 < 0) {
      out->push_back({a, z, false, (int32_t)(((int64_t)c + 1 + q) % p.N), p.N - q, true});
    } else {
      out->push_back({a, z, false, (int32_t)((e0 + q) % p.N), m - q, true});
    }
    a = z;
  }
}

// ---- transport executor helpers ---------------------------------------------------

// Pending fold segments of one dtype, launched together (multi-segment k_fold).
struct FoldBatch {
  std::vector<es::FoldSegDesc> segs;
  std::vector<std::vector<const void *>> src;
  es_dtype dt = ES_F32;
  uint64_t bytes = 0;
  bool empty() const { return segs.empty(); }
  es_status flush(es_handle h, cudaStream_t cs, float r) {
    if (segs.empty()) return ES_OK;
    const es::Plan &p = h->plan;
    for (size_t i = 0; i < segs.size(); ++i) segs[i].src = src[i].data();
    es_status st = h->timed(ES_KERNEL_FOLD, bytes, cs, [&](int *nl) {
      return es::launch_fold_multi(dt, p.N, r, p.compat, segs.data(), (int)segs.size(), cs, h->blocks_ov,
                                   h->threads_ov, nl);
    });
    segs.clear();
    src.clear();
    bytes = 0;
    return st;
  }
};

// Where a bucket's operands live for the transport schedules (G == 1, DIRECT,
// CHAIN): local contributions (slot or BORROWed buffer), DIRECT staging for
// remote ones, CHAIN partial buffers, the caller's output.
struct BucketAddr {
  es_handle h;
  const es::Plan &p;
  int32_t bucket;
  const es::BucketPlan &b;
  uint32_t esz;
  unsigned char *outp;
  bool inc;   // NEXT-1: every local EST folded its prefix at its stash this step
  BucketAddr(es_handle hh, int32_t bk, void *out)
      : h(hh), p(hh->plan), bucket(bk), b(hh->plan.bp[bk]), esz(hh->plan.bp[bk].esize),
        outp(reinterpret_cast<unsigned char *>(out)),
        inc((hh->plan.options & ES_OPT_INCREMENTAL) && hh->inc_next[bk] == hh->n_local) {}
  unsigned char *src_base(int32_t e) const {   // element 0 of local EST e's contribution
    const int32_t li = p.local_index[e];
    const void *bw = h->borrowed[(size_t)li * h->B + bucket];
    if (bw) return reinterpret_cast<unsigned char *>(const_cast<void *>(bw));
    return h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[bucket];
  }
  unsigned char *contrib_at(int32_t e, int64_t lo) const {
    if (p.local_index[e] >= 0) return src_base(e) + (uint64_t)lo * esz;
    return h->ws + p.stage_off + (uint64_t)b.stage_index[e] * b.stage_stride + (uint64_t)(lo - b.shard_lo) * esz;
  }
  unsigned char *part_at(int64_t id, int64_t lo) const {
    const es::Part &pt = b.parts[id];
    return h->ws + p.parts_off + b.part_base + pt.off + (uint64_t)(lo - pt.lo) * 4;
  }
  // The segments of FOLD op f restricted to [lo, hi) (a sub-range of the op's range).
  void fold(const int64_t *f, int64_t lo, int64_t hi, FoldBatch *out) const {
    if (hi <= lo) return;
    std::vector<Piece> pcs;   // NEXT-1: pieces continuing from the incremental partials
    inc_pieces(p, b, inc && f[5] == ES_BUF_NONE, lo, hi, f[3], (int32_t)f[4], &pcs);
    for (const Piece &pc : pcs) {
      const int64_t a = pc.lo;
      es::FoldSegDesc d;
      d.lo = a;
      d.n = pc.hi - a;
      d.C = (uint32_t)b.C;
      std::vector<const void *> src;
      if (pc.rot) {
        d.rot = true;
        for (int32_t e = 0; e < p.N; ++e) src.push_back(contrib_at(e, a));
      } else {
        d.rot = false;
        d.m = pc.m;
        for (int32_t t = 0; t < d.m; ++t) src.push_back(contrib_at((int32_t)((pc.e0 + t) % p.N), a));
      }
      if (f[5] == ES_BUF_PART) d.part_in = reinterpret_cast<const float *>(part_at(f[6], a));
      else if (pc.part) d.part_in = reinterpret_cast<const float *>(h->ws + p.inc_off + p.inc_bucket_off[bucket]) + a;
      d.out_partial = f[7] == ES_BUF_PART;
      d.out = d.out_partial ? (void *)part_at(f[8], a) : (void *)(outp + (uint64_t)a * esz);
      out->bytes += (uint64_t)d.n * ((uint64_t)src.size() * esz + (d.part_in ? 4 : 0) + (d.out_partial ? 4 : esz));
      out->segs.push_back(d);
      out->src.push_back(std::move(src));
    }
  }
  // SEND / RECV op f restricted to [lo, hi), posted into the open transport group.
  es_status xfer(const int64_t *f, int64_t lo, int64_t hi) const {
    if (hi <= lo) return ES_OK;
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
    es_status s = f[0] == ES_OP_SEND ? h->tp->send(ptr, nbytes, (int)f[3]) : h->tp->recv(ptr, nbytes, (int)f[3]);
    return s == ES_OK ? ES_OK : h->poison(s, h->tp->err);
  }
};

// CHAIN over a transport, tile-pipelined.  Every chunk is cut
// into W tiles (W from the call's largest chunk, <= 8, ~2^20 elements; the
// same on every rank).  Fold F(r, w) -- round r's segments restricted to tile
// w -- runs on the caller's stream; transfer T(r, w) -- round r's outgoing
// partials and round r+1's incoming ones, tile w -- is one transport group on
// the handle's side stream, after F(r, w); F(r+1, w) waits for T(r, w).  Both
// streams walk (r, w) in wavefront order (r + w ascending, r ascending), so
// every rank posts the same group sequence and the per-peer message order of
// the round executor is kept tile by tile; T(r, w) overlaps F(0, w+1),
// F(1, w), ...  The all-gather follows as one group on the caller's stream.
constexpr int64_t kChainTileElems = 1 << 20;
constexpr int64_t kChainMaxTiles = 8;

es_status chain_pipelined(es_handle h, const std::vector<int32_t> &bks, const std::vector<void *> &outs,
                          cudaStream_t cs, float r) {
  const es::Plan &p = h->plan;
  es_status s;
  if (!h->side && cudaStreamCreateWithFlags(&h->side, cudaStreamNonBlocking) != cudaSuccess)
    return h->poison(ES_ECUDA, "cudaStreamCreateWithFlags failed");
  uint64_t Cmax = 0;
  int32_t R = 0;
  for (int32_t bk : bks) {
    Cmax = std::max(Cmax, p.bp[bk].C);
    for (int32_t rr : p.bp[bk].op_round) R = std::max(R, rr + 1);
  }
  const int64_t W = std::max<int64_t>(1, std::min<int64_t>(kChainMaxTiles, ((int64_t)Cmax + kChainTileElems - 1) /
                                                                             kChainTileElems));
  auto tile = [&](int64_t lo, int64_t hi, int64_t w, int64_t *a, int64_t *z) {
    const int64_t per = ((hi - lo + W - 1) / W + p.A - 1) / p.A * p.A;   // A-aligned: fold needs lo % 8 == 0
    *a = std::min(hi, lo + w * per);
    *z = std::min(hi, lo + (w + 1) * per);
  };
  const size_t nev = 2 * (size_t)R * (size_t)W + 2;
  while (h->chain_ev.size() < nev) {
    cudaEvent_t e = nullptr;
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
      return h->poison(ES_ECUDA, "cudaEventCreate failed");
    h->chain_ev.push_back(e);
  }
  cudaEvent_t *FE = h->chain_ev.data(), *TE = FE + (size_t)R * W, *start = TE + (size_t)R * W, *join = start + 1;
  std::vector<uint8_t> te_used((size_t)R * W, 0);
  std::vector<BucketAddr> ad;
  ad.reserve(bks.size());
  for (size_t i = 0; i < bks.size(); ++i) ad.emplace_back(h, bks[i], outs[i]);
  // the side stream starts after everything before this call on the caller's stream
  if (cudaEventRecord(*start, cs) != cudaSuccess || cudaStreamWaitEvent(h->side, *start, 0) != cudaSuccess)
    return h->poison(ES_ECUDA, "event record / wait failed");
  for (int64_t d = 0; d < R + W - 1; ++d)
    for (int32_t rr = 0; rr < R; ++rr) {
      const int64_t w = d - rr;
      if (w < 0 || w >= W) continue;
      const size_t ix = (size_t)rr * W + w;
      if (rr > 0 && te_used[ix - W] && cudaStreamWaitEvent(cs, TE[ix - W], 0) != cudaSuccess)
        return h->poison(ES_ECUDA, "cudaStreamWaitEvent failed");
      for (int dd = 0; dd < 2; ++dd) {           // F(rr, w)
        FoldBatch fb;
        fb.dt = (es_dtype)dd;
        for (const BucketAddr &a : ad) {
          if ((int)a.b.dtype != dd) continue;
          for (size_t k = 0; k < a.b.ops.size(); ++k) {
            const int64_t *f = a.b.ops[k].f;
            if (f[0] != ES_OP_FOLD || a.b.op_round[k] != rr) continue;
            int64_t lo, hi;
            tile(f[1], f[2], w, &lo, &hi);
            a.fold(f, lo, hi, &fb);
          }
        }
        if ((s = fb.flush(h, cs, r)) != ES_OK) return s;
      }
      bool any = false;                          // T(rr, w)
      for (const BucketAddr &a : ad)
        for (size_t k = 0; k < a.b.ops.size() && !any; ++k) {
          const int64_t *f = a.b.ops[k].f;
          if ((f[0] == ES_OP_SEND || f[0] == ES_OP_RECV) && a.b.op_round[k] == rr) {
            int64_t lo, hi;
            tile(f[1], f[2], w, &lo, &hi);
            any = hi > lo;
          }
        }
      if (!any) continue;
      if (cudaEventRecord(FE[ix], cs) != cudaSuccess || cudaStreamWaitEvent(h->side, FE[ix], 0) != cudaSuccess)
        return h->poison(ES_ECUDA, "event record / wait failed");
      if ((s = h->tp->group_begin()) != ES_OK) return h->poison(s, h->tp->err);
      for (const BucketAddr &a : ad)
        for (size_t k = 0; k < a.b.ops.size(); ++k) {
          const int64_t *f = a.b.ops[k].f;
          if ((f[0] != ES_OP_SEND && f[0] != ES_OP_RECV) || a.b.op_round[k] != rr) continue;
          int64_t lo, hi;
          tile(f[1], f[2], w, &lo, &hi);
          if ((s = a.xfer(f, lo, hi)) != ES_OK) return s;
        }
      if ((s = h->tp->group_end(h->side)) != ES_OK) return h->poison(s, h->tp->err);
      if (cudaEventRecord(TE[ix], h->side) != cudaSuccess) return h->poison(ES_ECUDA, "cudaEventRecord failed");
      te_used[ix] = 1;
    }
  // join the side stream back, then the all-gather of every chain bucket as one group
  if (cudaEventRecord(*join, h->side) != cudaSuccess || cudaStreamWaitEvent(cs, *join, 0) != cudaSuccess)
    return h->poison(ES_ECUDA, "event record / wait failed");
  if ((s = h->tp->group_begin()) != ES_OK) return h->poison(s, h->tp->err);
  for (const BucketAddr &a : ad)
    for (size_t k = 0; k < a.b.ops.size(); ++k) {
      const int64_t *f = a.b.ops[k].f;
      if ((f[0] == ES_OP_SEND || f[0] == ES_OP_RECV) && a.b.op_round[k] < 0 && (s = a.xfer(f, f[1], f[2])) != ES_OK)
        return s;
    }
  if ((s = h->tp->group_end(cs)) != ES_OK) return h->poison(s, h->tp->err);
  return ES_OK;
}

es_status peer_barrier(es_handle h, cudaStream_t cs) {
  const es::Plan &p = h->plan;
  std::vector<uint64_t *> pf(p.G);
  for (int32_t g = 0; g < p.G; ++g) pf[g] = reinterpret_cast<uint64_t *>(h->peer_ws[g] + p.flags_off);
  return h->timed(ES_KERNEL_BARRIER, 0, cs, [&](int *nl) {
    *nl = 1;
    return es::launch_peer_barrier(pf.data(), reinterpret_cast<uint64_t *>(h->ws + p.flags_off), p.G, p.rank, cs);
  });
}

// Peer-memory schedules (PEER, PEER_CHAIN), phase-merged over the batch.
// Every bucket's op list is cut at its BARRIER ops into phases; phase k of
// all buckets runs as one fold launch and one gather launch per dtype, then
// one device barrier.  All ranks plan the same barrier count per bucket, so
// the merged sequence of barriers matches across ranks.
es_status peer_allreduce(es_handle h, int32_t n, const int32_t *buckets, void *const *outs, cudaStream_t cs, float r) {
  const es::Plan &p = h->plan;
  if (!h->peer_open) return set_err(ES_ESTATE, "peer-memory schedules need es_peer_open before es_allreduce");
  const bool pipe = !(p.options & ES_OPT_PEER_ROUNDS) && p.compat == 0;
  es_status s;
  auto inc_done = [&](int32_t bk) { return (p.options & ES_OPT_INCREMENTAL) && h->inc_next[bk] == h->n_local; };
  auto slot_of = [&](int32_t rank, int32_t e, int32_t b) {
    return h->peer_ws[rank] + p.grad_off + (uint64_t)p.owner_index[e] * p.slot_block + p.slot_off[b];
  };
  // 1. PEER buckets: peers read the ranges of BORROWed contributions outside
  //    our shard from the slot (PEER_CHAIN reads only local contributions).
  for (int dd = 0; dd < 2; ++dd) {
    std::vector<es::StashSegDesc> segs;
    uint64_t nbytes = 0;
    for (int32_t i = 0; i < n; ++i) {
      const es::BucketPlan &b = p.bp[buckets[i]];
      if ((int)b.dtype != dd || b.L == 0 || b.sched != ES_SCHED_PEER) continue;
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
  // 2. phases.  Tile-pipelined (default): every bucket runs as three
  //    phases -- [barrier] all folds (PEER: one shard fold; PEER_CHAIN: every
  //    round in k_fold_pipe, ordered by per-tile flags) [barrier] gathers --
  //    so a phase index is mapped: PEER_CHAIN folds of any round -> phase 1,
  //    gathers -> phase 2.  Otherwise phase k = the ops after the k-th barrier.
  int32_t phases = 0;
  for (int32_t i = 0; i < n; ++i) {
    int32_t k = 0;
    for (const es::Op &op : p.bp[buckets[i]].ops) k += op.f[0] == ES_OP_BARRIER;
    phases = std::max(phases, k + 1);
  }
  if (pipe) phases = std::min(phases, 3);
  auto phase_of = [&](const es::BucketPlan &b, int32_t k, int64_t op) -> int32_t {
    if (!pipe || b.sched != ES_SCHED_PEER_CHAIN) return k;
    return op == ES_OP_GATHER ? 2 : 1;
  };
  // ES_OPT_PEER_PUSH: buckets whose final results come out of k_fold (not k_fold_pipe) push them
  // into every peer's RESULT area; their gathers then read the own RESULT area.
  auto pushes = [&](const es::BucketPlan &b) -> bool {
    // (sources + push pointers of one segment must fit one launch's 1024-pointer table; the rule
    //  depends only on N and G, so every rank decides alike)
    return (p.options & ES_OPT_PEER_PUSH) && p.G > 1 && p.N + p.G - 1 <= 1024 &&
           (b.sched == ES_SCHED_PEER || (b.sched == ES_SCHED_PEER_CHAIN && !pipe));
  };
  std::vector<std::vector<void *>> push_ptrs;   // per fold segment; outlives the launches below
  for (int32_t ph = 0; ph < phases; ++ph) {
    for (int dd = 0; dd < 2; ++dd) {
      std::vector<es::FoldSegDesc> folds;
      std::vector<std::vector<const void *>> srcs;
      std::vector<es::StashSegDesc> gathers;
      std::vector<std::pair<int32_t, es::PipeSegDesc>> pipes;   // (round, segment)
      uint64_t fbytes = 0, pbytes = 0, gbytes = 0;
      for (int32_t i = 0; i < n; ++i) {
        const int32_t bk = buckets[i];
        const es::BucketPlan &b = p.bp[bk];
        if ((int)b.dtype != dd) continue;
        const uint32_t esz = b.esize;
        int32_t k = 0;
        for (const es::Op &op : b.ops) {
          const int64_t *f = op.f;
          if (f[0] == ES_OP_BARRIER) {
            ++k;
            continue;
          }
          if (phase_of(b, k, f[0]) != ph) continue;
          const int64_t lo = f[1], hi = f[2];
          if (f[0] == ES_OP_GATHER) {
            const int32_t from = pushes(b) ? p.rank : (int32_t)f[3];   // pushed: already in our RESULT
            gathers.push_back({h->peer_ws[from] + p.result_off + p.slot_off[bk] + (uint64_t)lo * esz,
                               reinterpret_cast<unsigned char *>(outs[i]) + (uint64_t)lo * esz, hi - lo});
            gbytes += 2 * (uint64_t)(hi - lo) * esz;
            continue;
          }
          // ES_OP_FOLD (NEXT-1: pieces continuing from the incremental partials)
          std::vector<Piece> pcs;
          inc_pieces(p, b, inc_done(bk) && f[5] == ES_BUF_NONE, lo, hi, f[3], (int32_t)f[4], &pcs);
          for (const Piece &pc : pcs) {
          es::FoldSegDesc d;
          d.lo = pc.lo;
          d.n = pc.hi - pc.lo;
          d.C = (uint32_t)b.C;
          std::vector<const void *> src;
          auto contrib = [&](int32_t e) -> const unsigned char * {
            const int32_t li = p.local_index[e];
            const void *bw = li >= 0 ? h->borrowed[(size_t)li * h->B + bk] : nullptr;
            const unsigned char *base = bw ? reinterpret_cast<const unsigned char *>(bw)
                                           : slot_of(p.est_to_gpu[e], e, bk);   // local or peer slot
            return base + (uint64_t)pc.lo * esz;
          };
          if (pc.rot) {
            d.rot = true;
            for (int32_t e = 0; e < p.N; ++e) src.push_back(contrib(e));
          } else {
            d.rot = false;
            d.m = pc.m;
            for (int32_t t = 0; t < d.m; ++t) src.push_back(contrib((int32_t)((pc.e0 + t) % p.N)));
          }
          if (f[5] == ES_BUF_PEER_PART)         // the previous GPU's partial, over NVLink
            d.part_in = reinterpret_cast<const float *>(h->peer_ws[f[6]] + p.peer_parts_off + b.peer_part_base +
                                                        (uint64_t)f[9]);
          else if (pc.part)                     // NEXT-1: this rank's incremental partial
            d.part_in = reinterpret_cast<const float *>(h->ws + p.inc_off + p.inc_bucket_off[bk]) + pc.lo;
          d.out_partial = f[7] == ES_BUF_PART;
          d.out = d.out_partial ? (void *)(h->ws + p.peer_parts_off + b.peer_part_base + (uint64_t)f[8])
                                : (void *)(h->ws + p.result_off + p.slot_off[bk] + (uint64_t)pc.lo * esz);
          if (!d.out_partial && pushes(b)) {
            std::vector<void *> dst;
            for (int32_t g = 0; g < p.G; ++g)
              if (g != p.rank) dst.push_back(h->peer_ws[g] + p.result_off + p.slot_off[bk] + (uint64_t)pc.lo * esz);
            push_ptrs.push_back(std::move(dst));
            d.push = push_ptrs.back().data();
            d.npush = (int32_t)push_ptrs.back().size();
          }
          const uint64_t nbytes =
              (uint64_t)d.n * ((uint64_t)src.size() * esz + (d.part_in ? 4 : 0) + (d.out_partial ? 4 : esz) +
                               (uint64_t)d.npush * esz);
          d.src = src.data();                     // the buffer survives the move below
          srcs.push_back(std::move(src));
          if (pipe && b.sched == ES_SCHED_PEER_CHAIN) {
            const int32_t rd = k - 1;                     // round of this segment
            const uint64_t c = (uint64_t)pc.lo / b.C;     // its chunk (segments span whole chunks)
            auto flag = [&](unsigned char *base, int32_t round) {
              return reinterpret_cast<uint64_t *>(base + p.pipe_flags_off) + b.pipe_flag_base +
                     (c * (uint64_t)b.chain_rounds + (uint64_t)round) * b.tiles_per_chunk;
            };
            es::PipeSegDesc q;
            q.f = d;
            q.wait = f[5] == ES_BUF_PEER_PART ? flag(h->peer_ws[f[6]], rd - 1) : nullptr;
            q.pub = d.out_partial ? flag(h->ws, rd) : nullptr;
            pipes.push_back({rd, q});
            pbytes += nbytes;
          } else {
            folds.push_back(d);
            fbytes += nbytes;
          }
          }
        }
      }
      if (!folds.empty()) {
        s = h->timed(ES_KERNEL_FOLD, fbytes, cs, [&](int *nl) {
          return es::launch_fold_multi((es_dtype)dd, p.N, r, p.compat, folds.data(), (int)folds.size(), cs,
                                       h->blocks_ov, h->threads_ov, nl);
        });
        if (s != ES_OK) return s;
      }
      if (!pipes.empty()) {
        // round-major order across buckets: k_fold_pipe's forward-progress rule
        std::stable_sort(pipes.begin(), pipes.end(), [](const auto &x, const auto &y) { return x.first < y.first; });
        std::vector<es::PipeSegDesc> segs;
        for (auto &q : pipes) segs.push_back(q.second);
        s = h->timed(ES_KERNEL_FOLD, pbytes, cs, [&](int *nl) {
          return es::launch_fold_pipe((es_dtype)dd, p.N, r, segs.data(), (int)segs.size(),
                                      reinterpret_cast<const uint64_t *>(h->ws + p.flags_off) + es::kEpochSlot,
                                      reinterpret_cast<unsigned int *>(
                                          reinterpret_cast<uint64_t *>(h->ws + p.flags_off) + es::kTicketSlot),
                                      h->peer_share, cs, nl);
        });
        if (s != ES_OK) return s;
      }
      if (!gathers.empty()) {
        s = h->timed(ES_KERNEL_GATHER, gbytes, cs, [&](int *nl) {
          return es::launch_stash_multi((es_dtype)dd, (es_dtype)dd, gathers.data(), (int)gathers.size(), cs,
                                        h->blocks_ov, h->threads_ov, nl);
        });
        if (s != ES_OK) return s;
      }
    }
    if (ph + 1 < phases && (s = peer_barrier(h, cs)) != ES_OK) return s;
  }
  return ES_OK;
}
}  // namespace

es_status es_allreduce_many(es_handle h, int32_t n, const int32_t *buckets, void *const *outs, es_stream stream) {
  ES_NVTX();
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
    if (h->inc_next[buckets[i]] != 0 && h->inc_next[buckets[i]] != h->n_local)
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
  FoldBatch pend;
  // CHAIN buckets run tile-pipelined (chain_pipelined) unless ES_OPT_PEER_ROUNDS; every rank
  // splits the call alike (the schedule per bucket is global), so messages still match.
  const bool chain_pipe = p.G > 1 && !(p.options & ES_OPT_PEER_ROUNDS);
  std::vector<int32_t> chain_i;

  for (int32_t i = 0; i < n; ++i) {
    const int32_t bucket = buckets[i];
    const es::BucketPlan &b = p.bp[bucket];
    if (chain_pipe && b.sched == ES_SCHED_CHAIN) {
      if (b.L > 0) chain_i.push_back(i);
      continue;
    }
    const BucketAddr ad(h, bucket, outs[i]);
    for (const es::Op &op : b.ops) {
      const int64_t *f = op.f;
      switch (f[0]) {
        case ES_OP_FOLD:
          if (!pend.empty() && pend.dt != b.dtype && (s = pend.flush(h, cs, r)) != ES_OK) return s;
          pend.dt = b.dtype;
          ad.fold(f, f[1], f[2], &pend);
          break;
        case ES_OP_GROUP_BEGIN:
          if ((s = pend.flush(h, cs, r)) != ES_OK) return s;
          if ((s = h->tp->group_begin()) != ES_OK) return h->poison(s, h->tp->err);
          break;
        case ES_OP_GROUP_END:
          if ((s = h->tp->group_end(cs)) != ES_OK) return h->poison(s, h->tp->err);
          break;
        case ES_OP_SEND:
        case ES_OP_RECV:
          if ((s = ad.xfer(f, f[1], f[2])) != ES_OK) return s;
          break;
        default:
          return h->poison(ES_ESTATE, "corrupt plan: bad opcode");
      }
    }
  }
  if ((s = pend.flush(h, cs, r)) != ES_OK) return s;
  if (!chain_i.empty()) {
    std::vector<int32_t> cb;
    std::vector<void *> co;
    for (int32_t i : chain_i) {
      cb.push_back(buckets[i]);
      co.push_back(outs[i]);
    }
    if ((s = chain_pipelined(h, cb, co, cs, r)) != ES_OK) return s;
  }
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


}  // extern "C"
