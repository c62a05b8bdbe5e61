// api_stash.cpp -- C ABI: the stash (a1), fused stash + context switch, and the
// NEXT-1 incremental fold.
#include <unistd.h>

#include "handle.h"

extern "C" {

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
        const bool early = follows_own_stash(h, cs);
        s = h->timed(ES_KERNEL_STASH, nbytes + (sw ? swap_bytes : 0), cs, [&](int *nl) {
          return es::launch_stash_multi((es_dtype)sd, (es_dtype)dd, segs.data(), (int)segs.size(), cs, h->switch_blocks(),
                                        h->switch_threads(), nl, sw, early, h->background());
        });
        if (s != ES_OK) return s;
        remember_stash_node(h, cs);
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
  ES_NVTX();
  return stash_impl(h, est, n, buckets, grads, gdts, mode, -1, stream);
}

es_status es_stash_fold_grads(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                              const es_dtype *gdts, es_stash_mode mode, es_stream stream) {
  ES_NVTX();
  es_status s = check_handle(h);
  if (s != ES_OK) return s;
  const es::Plan &p = h->plan;
  if (!(p.options & ES_OPT_INCREMENTAL))
    return set_err(ES_EUNSUPPORTED, "es_stash_fold_grads needs ES_OPT_INCREMENTAL");
  if (n < 0 || (n > 0 && (!buckets || !grads || !gdts))) return set_err(ES_EINVAL, "bad bucket/grad arrays");
  if (est < 0 || est >= p.N) return set_err(ES_EINVAL, "est out of range");
  if (mode != ES_STASH_COPY && mode != ES_STASH_BORROW) return set_err(ES_EINVAL, "mode must be COPY or BORROW");
  const int32_t li = p.local_index[est];
  if (li < 0) return set_err(ES_ESTATE, "est is not mapped to this rank");
  for (int32_t i = 0; i < n; ++i) {
    const int32_t bk = buckets[i];
    if (bk < 0 || bk >= h->B) return set_err(ES_EINVAL, "bucket out of range");
    const es::BucketPlan &b = p.bp[bk];
    if (gdts[i] != b.dtype) return set_err(ES_EINVAL, "incremental fold needs grad dtype == bucket dtype");
    if (b.L > 0 && (!grads[i] || !aligned16(grads[i])))
      return set_err(ES_EINVAL, "grad must be a 16-byte aligned device pointer");
    for (int32_t j = 0; j < i; ++j)
      if (buckets[j] == bk) return set_err(ES_EINVAL, "bucket listed twice");
    if (h->inc_next[bk] != li)
      return set_err(ES_ESTATE, "incremental fold expects the local ESTs of a bucket in ascending order");
    if (li == 0)
      for (int32_t lj = 0; lj < h->n_local; ++lj)
        if (h->stashed[(size_t)lj * h->B + bk])
          return set_err(ES_ESTATE, "bucket already stashed this step with es_stash_grad(s)");
  }
  cudaStream_t cs = reinterpret_cast<cudaStream_t>(stream);
  const unsigned long long cap = capture_id(cs);
  for (int32_t i = 0; i < n; ++i) {
    const int32_t bk = buckets[i];
    if (h->ar_recorded[bk] && h->ar_cap[bk] == cap && cudaStreamWaitEvent(cs, h->ar_ev[bk], 0) != cudaSuccess)
      return h->poison(ES_ECUDA, "cudaStreamWaitEvent failed");
  }
  const float r = 1.0f / (float)p.N;
  std::vector<uint8_t> folded(n, 0);
  for (int dd = 0; dd < 2; ++dd) {
    // (i) fold x_est into the partials of the chunks whose planned prefix holds it
    //     (plan_incremental): est is position t of the sequence first, first+1, ...
    std::vector<es::FoldSegDesc> segs;
    std::vector<std::vector<const void *>> srcs;
    uint64_t fbytes = 0;
    // (ii) stash the rest: what the end fold, the exchange or peers still read
    std::vector<es::StashSegDesc> st;
    uint64_t sbytes = 0;
    for (int32_t i = 0; i < n; ++i) {
      const int32_t bk = buckets[i];
      const es::BucketPlan &b = p.bp[bk];
      if ((int)b.dtype != dd || b.L == 0) continue;
      const unsigned char *x = reinterpret_cast<const unsigned char *>(grads[i]);
      float *part = reinterpret_cast<float *>(h->ws + p.inc_off + p.inc_bucket_off[bk]);
      std::vector<std::pair<int64_t, int64_t>> used;   // ranges consumed here, ascending
      for (const es::IncChunk &ic : b.inc) {
        const int32_t t = (int32_t)(((int64_t)est - ic.first + p.N) % p.N);
        if (t >= ic.q) continue;
        const bool cont = t > 0;                 // t == 0: est opens the partial (c+1)
        // adjacent ranges with the same continuation merge into one segment
        if (!segs.empty() && srcs.back()[0] == (const void *)(x + (uint64_t)segs.back().lo * b.esize) &&
            segs.back().lo + segs.back().n == ic.lo && (segs.back().part_in != nullptr) == cont) {
          segs.back().n += ic.hi - ic.lo;
        } else {
          es::FoldSegDesc d;
          d.lo = ic.lo;
          d.n = ic.hi - ic.lo;
          d.C = (uint32_t)b.C;
          d.rot = false;
          d.m = 1;
          d.part_in = cont ? part + ic.lo : nullptr;
          d.out_partial = true;
          d.out = part + ic.lo;
          segs.push_back(d);
          srcs.push_back({x + (uint64_t)ic.lo * b.esize});
        }
        fbytes += (uint64_t)(ic.hi - ic.lo) * (b.esize + (cont ? 8 : 4));
        if (!used.empty() && used.back().second == ic.lo) used.back().second = ic.hi;
        else used.push_back({ic.lo, ic.hi});
      }
      folded[i] = !used.empty();
      if (mode == ES_STASH_COPY) {
        unsigned char *slot = h->ws + p.grad_off + (uint64_t)li * p.slot_block + p.slot_off[bk];
        int64_t at = 0;
        used.push_back({(int64_t)b.L, (int64_t)b.L});
        for (const auto &u : used) {
          if (u.first > at) {
            st.push_back({x + (uint64_t)at * b.esize, slot + (uint64_t)at * b.esize, u.first - at});
            sbytes += 2 * (uint64_t)(u.first - at) * b.esize;
          }
          at = u.second;
        }
      }
    }
    if (!segs.empty()) {
      for (size_t j = 0; j < segs.size(); ++j) segs[j].src = srcs[j].data();
      s = h->timed(ES_KERNEL_FOLD, fbytes, cs, [&](int *nl) {
        return es::launch_fold_multi((es_dtype)dd, p.N, r, p.compat, segs.data(), (int)segs.size(), cs,
                                     h->switch_blocks(), h->switch_threads(), nl);
      });
      if (s != ES_OK) return s;
    }
    if (!st.empty()) {
      s = h->timed(ES_KERNEL_STASH, sbytes, cs, [&](int *nl) {
        return es::launch_stash_multi((es_dtype)dd, (es_dtype)dd, st.data(), (int)st.size(), cs,
                                      h->switch_blocks(), h->switch_threads(), nl, nullptr, false,
                                      h->background());
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
    h->inc_next[buckets[i]] = li + 1;
    // the slot holds the whole gradient iff nothing of it was folded here
    h->inc_full[k] = mode == ES_STASH_COPY && !folded[i] ? 1 : 0;
  }
  return ES_OK;
}

es_status es_stash_and_switch(es_handle h, int32_t est, int32_t n, const int32_t *buckets, const void *const *grads,
                              const es_dtype *gdts, es_stash_mode mode, int32_t next_est, es_stream stream) {
  ES_NVTX();
  if (next_est < 0) return set_err(ES_EINVAL, "next_est must be a valid EST (use es_stash_grads to only stash)");
  return stash_impl(h, est, n, buckets, grads, gdts, mode, next_est, stream);
}

es_status es_stash_grad(es_handle h, int32_t est, int32_t bucket, const void *grad, es_dtype gdt, es_stash_mode mode,
                        es_stream stream) {
  ES_NVTX();
  return stash_impl(h, est, 1, &bucket, &grad, &gdt, mode, -1, stream);
}


}  // extern "C"
