#!/usr/bin/env python
"""Exposed aggregation time when the stash overlaps training compute (G = 1).

The paper hides the gradient swap behind the next EST's forward pass and
triggers the synchronisation after the last EST (PAPER.md:599-606,
PAPER.md:1287-1296).  bench.py times the hot path alone, with nothing to hide
behind; this probe puts a synthetic training step around it and measures what
is left exposed.

Per EST k, on a compute stream: es_switch_context(k), a "forward" of bf16
GEMMs (a stand-in for the model's compute; cuBLAS, not part of the hot path),
a "backward" of twice as many GEMMs, then the gradient write of all buckets
(EST k's synthetic gradients copied into the live gradient buffer, or into
EST k's slot for the zero-copy mode).  On an aggregation stream, once EST k's
gradients are written: its stash (mode below).  The live buffer is reused by
the next EST, so EST k+1's gradient write waits for EST k's stash.  After the
last EST: es_allreduce_many on the aggregation stream, joined back.

modes: base[+flag...]
  none         compute + gradient writes only (the floor)
  copy         the paper's step: ESTs 0..N-2 ES_STASH_COPY, EST N-1 BORROW
  incremental  NEXT-1 es_stash_fold_grads (last EST's fold deferred to the end fold)
  inplace      NEXT-2 zero-copy: gradients written into the slots, ES_STASH_INPLACE
  copy_serial  the copy stash on the compute stream (no overlap)
  copy_ce      diagnostic: the slot copy by cudaMemcpyAsync (copy engines, no
               SMs) on the aggregation stream, then ES_STASH_INPLACE
flags
  +bk          DDP-style buckets (copy / inplace): the backward is split into one slice per bucket
               and bucket b's gradient is written after its slice (buckets are in reverse layer
               order, as DDP fills them); each bucket is stashed as soon as it is written, and for
               the last EST es_allreduce(b) is launched as soon as its bucket b is written, so the
               folds of all but the last bucket overlap the last EST's backward
  +bg          ES_OPT_STASH_BACKGROUND (stash / incremental-fold grids of one wave)
  +lp          compute stream at high priority (the aggregation fills the gaps)
  +hp          aggregation stream at high priority
  +ovK         es_set_launch_override(148*K, 256): every libes launch (stash, fold) is a grid of
               K CTAs per SM (grid-stride), leaving SM slots to the compute stream

Reported per mode: step ms, exposed ms = median over rounds of (this mode's
median step - the compute-only median of the same round), tail ms = last gradient
written -> allreduce done (the critical path the aggregation adds).  The
reduced buckets of every mode are compared word for word with the first
aggregating mode's.  Modes run interleaved for --rounds rounds.

  python scripts/overlap_probe.py [--config resnet50] [--fwd-us 1000] [--steps 10]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="resnet50")
    ap.add_argument("--fwd-us", type=float, default=1000.0, help="synthetic forward per EST (backward = 2x)")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--rounds", type=int, default=6)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--compute", default="gemm", choices=["gemm", "sleep"],
                    help="gemm: cuBLAS bf16 GEMMs on every SM; sleep: a spin kernel (uncontended overlap)")
    ap.add_argument("--modes", default="none,copy,incremental,inplace")
    args = ap.parse_args()

    import torch
    from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads
    from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    cfg = workloads.config(args.config)
    N, buckets = cfg["N"], cfg["buckets"]
    B = len(buckets)
    src = [[workloads.est_bucket(args.config, k, b, device=dev) for b in range(B)] for k in range(N)]
    live = [torch.empty_like(src[0][b]) for b in range(B)]

    # synthetic compute: 4096^3 bf16 GEMMs, count calibrated to --fwd-us
    a = torch.randn(4096, 4096, device=dev, dtype=torch.bfloat16)
    w = torch.randn(4096, 4096, device=dev, dtype=torch.bfloat16)
    c = torch.empty(4096, 4096, device=dev, dtype=torch.bfloat16)
    for _ in range(10):
        torch.matmul(a, w, out=c)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(50):
        torch.matmul(a, w, out=c)
    e1.record()
    torch.cuda.synchronize()
    gemm_us = e0.elapsed_time(e1) * 1e3 / 50
    n_fwd = max(1, round(args.fwd_us / gemm_us))

    # copy-engine D2D bandwidth (cudaMemcpyAsync via torch copy_ of contiguous same-dtype tensors)
    tmp = [torch.empty_like(x) for x in live]
    for x, y in zip(tmp, src[0]):
        x.copy_(y)
    e0.record()
    for _ in range(10):
        for x, y in zip(tmp, src[1]):
            x.copy_(y)
    e1.record()
    torch.cuda.synchronize()
    ce_gbps = 10 * 2 * sum(x.numel() * x.element_size() for x in tmp) / (e0.elapsed_time(e1) / 1e3) / 1e9
    del tmp
    cycles_per_us = torch.cuda.get_device_properties(dev).clock_rate / 1e3   # kHz -> cycles per us

    def compute(n):
        if args.compute == "sleep":      # one spinning thread: no SM or HBM contention at all
            torch.cuda._sleep(int(n * gemm_us * cycles_per_us))
            return
        for _ in range(n):
            torch.matmul(a, w, out=c)

    snb = workloads.state_nbytes()
    state = [torch.zeros(n, dtype=torch.uint8, device=dev) for n in snb]
    modes = args.modes.split(",")
    if "none" not in modes:
        modes = ["none"] + modes

    def make(mode):
        # mode = base[+flag...]; flags: bg = ES_OPT_STASH_BACKGROUND, lp = compute stream at
        # high priority (the aggregation fills gaps), hp = aggregation stream at high priority.
        # torch stream priority: -1 = high, 0 = default (low).
        base_mode, *flags = mode.split("+")
        sc = torch.cuda.Stream(device=dev, priority=-1 if "lp" in flags else 0)
        sa = torch.cuda.Stream(device=dev, priority=-1 if "hp" in flags else 0)
        if base_mode == "copy_serial":
            sa, base_mode = sc, "copy"
        opts = (es.ES_OPT_INCREMENTAL if base_mode == "incremental" else 0) | \
            (es.ES_OPT_STASH_BACKGROUND if "bg" in flags else 0)
        agg = Aggregator(N, 1, 0, [0] * N, buckets, state_nbytes=snb, device=dev,
                         options=opts)
        agg.register_state(state)
        for f in flags:                               # +ovK: every launch capped at K 256-thread CTAs per SM
            if f.startswith("ov"):
                agg.set_launch_override(148 * int(f[2:]), 256)
        for k in range(N):
            for i, blob in enumerate(workloads.est_state(args.config, k)):
                agg.init_state(k, i, blob)
        outs = [agg.new_out(b) for b in range(B)]
        slots = [[agg.slot(k, b) for b in range(B)] for k in range(N)]
        ev_grad = [torch.cuda.Event() for _ in range(N)]
        ev_stash = [torch.cuda.Event() for _ in range(N)]
        ev_done = torch.cuda.Event()
        # per EST: aggregation-stream busy time (stash start -> stash done), last step only
        ev_s0 = [torch.cuda.Event(enable_timing=True) for _ in range(N)]
        ev_s1 = [torch.cuda.Event(enable_timing=True) for _ in range(N)]
        # compute-stream time per EST (switch .. last gradient written), last step only
        ev_est = [torch.cuda.Event(enable_timing=True) for _ in range(N + 1)]

        bucketed = "bk" in flags and base_mode in ("copy", "inplace")
        n_bwd = 2 * n_fwd
        bwd_slices = [n_bwd * (j + 1) // B - n_bwd * j // B for j in range(B)]
        ev_gb = [[torch.cuda.Event() for _ in range(B)] for _ in range(N)]      # bucket written
        ev_sb = [[torch.cuda.Event() for _ in range(B)] for _ in range(N)]      # bucket stashed

        def step_bucketed(t0, t_last, t1):
            # DDP-style: per-bucket gradient readiness inside each EST's backward
            with torch.cuda.stream(sc):
                t0.record(sc)
                sc.wait_event(ev_done)
                for k in range(N):
                    last = k == N - 1
                    ev_est[k].record(sc)
                    agg.switch(k, stream=sc)
                    compute(n_fwd)
                    for b in range(B):
                        compute(bwd_slices[b])
                        if base_mode == "copy" and k > 0:
                            sc.wait_event(ev_sb[k - 1][b])           # EST k-1's bucket b left the live buffer
                        dst = slots[k][b] if base_mode == "inplace" else live[b]
                        dst.copy_(src[k][b])
                        ev_gb[k][b].record(sc)
                        with torch.cuda.stream(sa):
                            sa.wait_event(ev_gb[k][b])
                            if b == 0:
                                ev_s0[k].record(sa)
                            mode_b = es.ES_STASH_INPLACE if base_mode == "inplace" else \
                                (es.ES_STASH_BORROW if last else es.ES_STASH_COPY)
                            agg.stash_many(k, [b], [dst], mode_b, stream=sa)
                            ev_sb[k][b].record(sa)
                            if last:
                                agg.allreduce_many([b], [outs[b]], stream=sa)
                            if b == B - 1:
                                ev_s1[k].record(sa)
                ev_est[N].record(sc)
                t_last.record(sc)
                with torch.cuda.stream(sa):
                    ev_done.record(sa)
                sc.wait_event(ev_done)
                t1.record(sc)

        def step(t0, t_last, t1):
            if bucketed:
                return step_bucketed(t0, t_last, t1)
            with torch.cuda.stream(sc):
                t0.record(sc)
                sc.wait_event(ev_done)                # previous step's allreduce (BORROW / slots)
                for k in range(N):
                    ev_est[k].record(sc)
                    if base_mode != "none":
                        agg.switch(k, stream=sc)
                    compute(n_fwd)
                    for b in range(B):                        # the backward in B slices in every mode,
                        compute(bwd_slices[b])                # so +bk adds no kernel boundaries
                    if base_mode in ("copy", "incremental", "copy_ce") and k > 0:
                        sc.wait_event(ev_stash[k - 1])    # the live buffer is free again
                    dst = slots[k] if base_mode == "inplace" else live
                    for b in range(B):
                        dst[b].copy_(src[k][b])
                    ev_grad[k].record(sc)
                    if base_mode == "none":
                        continue
                    with torch.cuda.stream(sa):
                        sa.wait_event(ev_grad[k])
                        ev_s0[k].record(sa)
                        last = k == N - 1
                        if base_mode == "copy":
                            agg.stash_many(k, range(B), live, es.ES_STASH_BORROW if last else es.ES_STASH_COPY,
                                           stream=sa)
                        elif base_mode == "incremental":
                            agg.stash_fold(k, range(B), live, es.ES_STASH_BORROW if last else es.ES_STASH_COPY,
                                           stream=sa)
                        elif base_mode == "copy_ce" and not last:
                            for b in range(B):
                                slots[k][b].copy_(live[b])
                            agg.stash_many(k, range(B), slots[k], es.ES_STASH_INPLACE, stream=sa)
                        elif base_mode == "copy_ce":
                            agg.stash_many(k, range(B), live, es.ES_STASH_BORROW, stream=sa)
                        else:
                            agg.stash_many(k, range(B), dst, es.ES_STASH_INPLACE, stream=sa)
                        ev_stash[k].record(sa)
                        ev_s1[k].record(sa)
                ev_est[N].record(sc)
                t_last.record(sc)
                if base_mode != "none":
                    sa.wait_event(ev_grad[N - 1])
                    with torch.cuda.stream(sa):
                        agg.allreduce_many(range(B), outs, stream=sa)
                        ev_done.record(sa)
                    sc.wait_event(ev_done)
                t1.record(sc)
        def stash_ms():
            return sum(a.elapsed_time(b) for a, b in zip(ev_s0, ev_s1)) if base_mode != "none" else 0.0
        def est_ms():
            d = [ev_est[k].elapsed_time(ev_est[k + 1]) for k in range(N)]
            return [d[0], statistics.median(d[1:-1]) if N > 2 else 0.0, d[-1]]
        return {"agg": agg, "outs": outs, "step": step, "stash_ms": stash_ms, "est_ms": est_ms}

    ctx = {m: make(m) for m in modes}
    times = {m: [] for m in modes}
    stash_t = {}                   # (step, tail) per timed step
    est_t = {}                     # [first, median middle, last] EST compute-stream ms, last step per round
    for r in range(args.rounds):                     # modes interleaved: clock/power drift hits all alike
        for m in modes:
            ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.warmup + args.steps)]
            for i in range(args.warmup + args.steps):
                ctx[m]["step"](*ev[i])
            torch.cuda.synchronize()
            times[m] += [(e[0].elapsed_time(e[2]), e[1].elapsed_time(e[2])) for e in ev[args.warmup:]]
            stash_t.setdefault(m, []).append(ctx[m]["stash_ms"]())
            est_t.setdefault(m, []).append(ctx[m]["est_ms"]())
    results, ref = [], None

    def block_medians(m):
        v = [t for t, _ in times[m]]
        return [statistics.median(v[i:i + args.steps]) for i in range(0, len(v), args.steps)]
    base_r = block_medians("none")
    for m in modes:
        ctx[m]["agg"].sync()
        # exposed = per round, this mode's median step minus the compute-only median of the same round
        d = sorted(x - y for x, y in zip(block_medians(m), base_r))
        res = {"mode": m, "step_ms": round(statistics.median(t for t, _ in times[m]), 4),
               "exposed_ms": round(statistics.median(d), 4),
               "exposed_min_max_ms": [round(d[0], 4), round(d[-1], 4)],
               "tail_ms": round(statistics.median(t for _, t in times[m]), 4),
               "stash_stream_busy_ms": round(statistics.median(stash_t[m]), 4),
               "est_ms_first_mid_last": [round(statistics.median(e[i] for e in est_t[m]), 4) for i in range(3)]}
        if m != "none":
            got = ctx[m]["outs"]
            if ref is None:
                ref = got
            res["bits_equal_" + modes[1] + "_mode"] = all(torch.equal(x.view(torch.uint8), y.view(torch.uint8))
                                                         for x, y in zip(got, ref))
        results.append(res)
    print(json.dumps({"probe": "overlap", "config": args.config, "N": N, "G": 1, "compute": args.compute,
                      "gemm_us": round(gemm_us, 2), "memcpy_d2d_GBps_read_plus_write": round(ce_gbps, 1), "gemms_per_est": 3 * n_fwd,
                      "compute_ms_per_est": round(3 * n_fwd * gemm_us / 1e3, 3),
                      "payload_MB_per_step": round(workloads.payload_bytes(args.config) / 1e6, 1),
                      "rounds": args.rounds, "steps_per_round": args.steps, "modes": results}))


if __name__ == "__main__":
    main()
