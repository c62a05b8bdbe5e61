#!/usr/bin/env python
"""bench.py -- EST-gradient GB/s reduced (bit-exact across G), % of roofline.

One STEP = one global step of EasyScale's data-parallel hot path over one
batch of synthetic gradients: for every local EST
a context switch (k_swap over the Philox record + BN payload) and a stash of
each bucket (k_stash; the last local EST is borrowed),
then es_allreduce of every bucket (exchange + canonical fold + 1/N + gather).
value = N * sum_b L_b * bytes / step time (whole job; inputs resident in HBM).

  python bench.py [--gpus N --steps K --warmup W] [--config resnet50] [--impl reference]
  (N > 1: torchrun --nproc-per-node N ... bench.py --gpus N ...; NCCL transport)

Prints ONE JSON line on rank 0.  See DESIGN.md "Measurement".
"""
import argparse
import hashlib
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "EST-gradient GB/s reduced (bit-exact across G) at 1/2/4/8 B200; % of roofline"
L2_BYTES = 126 * 1024 * 1024
HBM_NOMINAL_GBPS = 8000.0     # B200 HBM3e nominal (SURVEY 8(d) t_roof uses 8.0 TB/s); `frac` uses the measured peak


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="es200", choices=["es200", "reference"])
    p.add_argument("--config", default="resnet50",
                   choices=["tiny", "resnet50", "vgg19", "bert_base", "swin_b"])
    p.add_argument("--mapping", default="contiguous", choices=["contiguous", "round_robin", "random"])
    p.add_argument("--sched", default=None, choices=["auto", "direct", "chain", "peer", "peer_chain", "peer_auto"],
                   help="default: auto at G=1; peer_auto at G>1 (fused folds over NVLink peer memory, CUDA IPC)")
    p.add_argument("--no-graph", action="store_true", help="eager launches instead of one CUDA graph per step")
    p.add_argument("--per-bucket", action="store_true",
                   help="one es_stash_grad / es_allreduce call per bucket (DDP-style) instead of the batched calls")
    p.add_argument("--no-fuse", action="store_true",
                   help="separate es_switch_context and es_stash_grads launches instead of es_stash_and_switch")
    p.add_argument("--incremental", action="store_true",
                   help="NEXT-1: fold each EST into running partials at its switch (es_stash_fold_grads, G == 1)")
    p.add_argument("--inplace", action="store_true",
                   help="NEXT-2 zero-copy stash: each EST's gradients are produced in its slot (es_slot_ptr) and "
                        "stashed with ES_STASH_INPLACE")
    p.add_argument("--stash-background", action="store_true",
                   help="ES_OPT_STASH_BACKGROUND: one-wave stash grids (for overlap with compute; scripts/overlap_probe.py)")
    p.add_argument("--peer-push", action="store_true",
                   help="ES_OPT_PEER_PUSH (G>1, peer schedules): the all-gather fused into the fold as NVLink stores")
    p.add_argument("--rehearse-same-gpu", action="store_true",
                   help="functional rehearsal of the N>1 path on ONE GPU: every rank on cuda:0, gloo process "
                        "group, a peer schedule (CUDA IPC, no NCCL); times are not GPU-scaling numbers")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    p.add_argument("--cpu-seconds", type=float, default=10.0)
    return p.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def cores_used():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count()


# ---- clocks sampler ------------------------------------------------------------------------

class Clocks:
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None
        self.t0 = time.time()

    def mark(self):
        return time.time()

    def stop(self, t_start, t_end):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.15)
        self.proc.terminate()
        self.proc.wait()
        self.f.flush()
        rows = []
        with open(self.f.name) as f:
            for line in f:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) >= 9:
                    rows.append(parts)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        # samples are ~50 ms apart; keep the ones during the timed window (+1 sample on each side)
        n = len(rows)
        total = max(time.time() - self.t0, 1e-3)
        lo = int(max(0, (t_start - self.t0) / total * n - 1))
        hi = int(min(n, (t_end - self.t0) / total * n + 2))
        win = rows[lo:hi] or rows
        sm = [float(r[1]) for r in win if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in win if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in win for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(win)}


# ---- oracle legs (cpu_baseline / --impl reference) -----------------------------------------

def oracle_windows(name, fetch, budget_s, seed=0):
    """Times the oracle, as it stands (single thread), on windows of every
    bucket until ~budget_s of CPU work.  fetch(k, b, s, n) -> EST k's bucket b
    elements [s, s+n) as numpy.  Returns (GB/s, sample text, [(b, s, n, out)])."""
    import numpy as np
    import oracle
    from paper_conf_sc_lixyszrljlllq23_b200 import workloads
    cfg = workloads.config(name)
    N = cfg["N"]
    esz = 2 if cfg["dtype"] == "bf16" else 4
    rng = np.random.default_rng(seed)
    done_bytes, t_oracle, windows = 0, 0.0, []
    win = 1 << 18
    t_begin = time.time()
    while t_oracle < budget_s and time.time() - t_begin < 3 * budget_s:
        for b, (L, d) in enumerate(cfg["buckets"]):
            n = min(win, L)
            s = int(rng.integers(0, L - n + 1))
            xs = [fetch(k, b, s, n) for k in range(N)]
            t0 = time.perf_counter()
            out = oracle.reduce(xs, d, L=L, first=s)
            t_oracle += time.perf_counter() - t0
            done_bytes += N * n * esz
            windows.append((b, s, n, out))
            if t_oracle >= budget_s:
                break
    gbs = done_bytes / t_oracle / 1e9
    sample = (f"{len(windows)} windows of <= {win} elements x {N} ESTs across the {len(cfg['buckets'])} buckets "
              f"({done_bytes / 1e6:.1f} MB of EST gradients, {t_oracle:.1f} s single-thread C oracle)")
    return gbs, sample, windows


def oracle_all_cores(name, fetch, threads, budget_s=3.0, max_bytes=512 << 20, seed=7):
    """The same unmodified single-thread oracle, one window per host thread at a
    time on every available core (ctypes releases the GIL inside the C call;
    each element's fold order is unchanged).  Inputs are fetched before the
    clock starts.  Returns (GB/s, sample text)."""
    import concurrent.futures as cf
    import numpy as np
    import oracle
    from paper_conf_sc_lixyszrljlllq23_b200 import workloads
    cfg = workloads.config(name)
    N = cfg["N"]
    esz = 2 if cfg["dtype"] == "bf16" else 4
    win = 1 << 18
    n_win = max(threads, min(4 * threads, max_bytes // (N * win * esz)))
    rng = np.random.default_rng(seed)
    jobs = []
    for j in range(n_win):
        b = j % len(cfg["buckets"])
        L, d = cfg["buckets"][b]
        n = min(win, L)
        s = int(rng.integers(0, L - n + 1))
        jobs.append(([fetch(k, b, s, n) for k in range(N)], d, L, s, N * n * esz))
    reps = 0
    with cf.ThreadPoolExecutor(max_workers=threads) as ex:
        t0 = time.perf_counter()
        while reps == 0 or time.perf_counter() - t0 < budget_s:     # the job list, repeated
            list(ex.map(lambda jb: oracle.reduce(jb[0], jb[1], L=jb[2], first=jb[3]), jobs))
            reps += 1
        dt = time.perf_counter() - t0
    done = reps * sum(jb[4] for jb in jobs)
    return done / dt / 1e9, (f"{reps} x {n_win} windows of <= {win} elements x {N} ESTs ({done / 1e6:.1f} MB of "
                             f"EST gradients) on {threads} threads, {dt:.2f} s wall")


def workload_config(args, cfg, G):
    """The `config` keys both arms share (the same workload)."""
    return {"workload": args.config, "N": cfg["N"], "G": G, "mapping": args.mapping, "sched": args.sched,
            "buckets": len(cfg["buckets"]), "elements": sum(n for n, _ in cfg["buckets"]), "desc": cfg["desc"]}


def run_reference(args, rank, world):
    if rank != 0:
        return
    from paper_conf_sc_lixyszrljlllq23_b200 import workloads
    name = args.config
    cfg = workloads.config(name)
    cache = {}

    def fetch(k, b, s, n):
        if (k, b) not in cache:
            t = workloads.est_bucket(name, k, b, device="cpu")
            cache[(k, b)] = t.numpy() if cfg["dtype"] == "f32" else t.view(__import__("torch").int16).numpy().view("uint16")
        return cache[(k, b)][s:s + n]

    # one "step" = one bounded sample of the workload; K timed samples after W warm-ups
    budget = max(0.5, min(args.cpu_seconds, 60.0 / max(1, args.steps + args.warmup)))
    for _ in range(args.warmup):
        oracle_windows(name, fetch, budget * 0.2, seed=1)
    rates, sample = [], ""
    for i in range(args.steps):
        gbs, sample, _ = oracle_windows(name, fetch, budget, seed=100 + i)
        rates.append(gbs)
    value = statistics.median(rates)
    payload = workloads.payload_bytes(name)
    ms = payload / (value * 1e9) * 1e3
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GB/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": cfg["dtype"], "data": "synthetic",
        "config": dict(workload_config(args, cfg, world), graph=False, api="C oracle (single thread)",
                       l2="host memory"),
        "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": sample + "; ms_per_step extrapolates the full step"},
        "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ---- the GPU arm ------------------------------------------------------------------------------

def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.sched is None:
        args.sched = "peer_auto" if world > 1 else "auto"
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads
    from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator, nccl_comm_ptr

    rehearse = args.rehearse_same_gpu and world > 1
    if rehearse and args.sched not in ("peer", "peer_chain", "peer_auto"):
        raise SystemExit("--rehearse-same-gpu needs --sched peer|peer_chain|peer_auto (NCCL refuses two ranks per GPU)")
    if rehearse:
        local_rank = 0
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    comm = None

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cpu" if rehearse else dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    if rehearse:
        dist.init_process_group("gloo")
    elif world > 1:
        dist.init_process_group("nccl", device_id=dev)
        t = torch.ones(1, device=dev)
        dist.all_reduce(t)                       # create the NCCL communicator
        torch.cuda.synchronize()
        comm = nccl_comm_ptr()
    name = args.config
    cfg = workloads.config(name)
    N, G = cfg["N"], world
    mapping = workloads.mapping(N, G, args.mapping)
    local = [k for k in range(N) if mapping[k] == rank]
    buckets = cfg["buckets"]
    B = len(buckets)
    sched = {"auto": es.ES_SCHED_AUTO, "direct": es.ES_SCHED_DIRECT, "chain": es.ES_SCHED_CHAIN,
             "peer": es.ES_SCHED_PEER, "peer_chain": es.ES_SCHED_PEER_CHAIN, "peer_auto": es.ES_SCHED_PEER_AUTO}[args.sched]
    snb = workloads.state_nbytes()
    agg = Aggregator(N, G, rank, mapping, buckets, state_nbytes=snb,
                     transport=es.ES_TRANSPORT_NONE if G == 1 or rehearse else es.ES_TRANSPORT_NCCL, comm=comm,
                     sched=sched,
                     device=dev, options=(es.ES_OPT_INCREMENTAL if args.incremental else 0) |
                     (es.ES_OPT_STASH_BACKGROUND if args.stash_background else 0) |
                     (es.ES_OPT_PEER_PUSH if args.peer_push else 0))
    if G > 1 and sched in es.PEER_SCHEDS:
        agg.peer_connect()                       # CUDA IPC map of every peer's workspace (NVLink)
    live = [torch.zeros(n, dtype=torch.uint8, device=dev) for n in snb]
    agg.register_state(live)
    for k in local:
        for i, blob in enumerate(workloads.est_state(name, k)):
            agg.init_state(k, i, blob)
    if args.inplace:       # the synthetic "backward" writes straight into the EST's slots
        grads = {k: [workloads.est_bucket(name, k, b, device=dev, out=agg.slot(k, b)) for b in range(B)]
                 for k in local}
    else:
        grads = {k: [workloads.est_bucket(name, k, b, device=dev) for b in range(B)] for k in local}
    outs = [agg.new_out(b) for b in range(B)]
    esz = 2 if cfg["dtype"] == "bf16" else 4
    in_bytes = len(local) * sum(n for n, _ in buckets) * esz
    flush = None if in_bytes > 2 * L2_BYTES else torch.empty(4 * L2_BYTES, dtype=torch.uint8, device=dev)
    if flush is not None:
        flush_words = flush.view(torch.int32)
        flush_sink = torch.zeros((), dtype=torch.int32, device=dev)
    torch.cuda.synchronize()

    fuse = not (args.per_bucket or args.no_fuse or args.incremental or args.inplace)

    def step(marks=None):
        # marks: three external CUDA events recorded at the phase boundaries
        # (stashes start | stashes done | allreduce done) of one captured step
        def mark(j):
            if marks is not None:
                marks[j].record(torch.cuda.current_stream())
        if args.inplace:
            agg.switch(local[0])
            mark(0)
            for i, k in enumerate(local):
                if i == len(local) - 1:
                    agg.stash_many(k, range(B), grads[k], es.ES_STASH_INPLACE)
                else:
                    agg.stash_and_switch(k, range(B), grads[k], local[i + 1], es.ES_STASH_INPLACE)
            mark(1)
            agg.allreduce_many(range(B), outs)
            mark(2)
            return
        if args.incremental:
            mark(0)
            for i, k in enumerate(local):
                agg.switch(k)
                agg.stash_fold(k, range(B), grads[k], es.ES_STASH_BORROW if i == len(local) - 1 else es.ES_STASH_COPY)
            mark(1)
            agg.allreduce_many(range(B), outs)
            mark(2)
            return
        if fuse:
            # switch-in of the first local EST, then per EST: stash its
            # buckets + switch to the next EST in one launch
            agg.switch(local[0])
            mark(0)
            for i, k in enumerate(local):
                if i == len(local) - 1:
                    agg.stash_many(k, range(B), grads[k], es.ES_STASH_BORROW)
                else:
                    agg.stash_and_switch(k, range(B), grads[k], local[i + 1], es.ES_STASH_COPY)
        if not fuse:
            mark(0)
        for i, k in enumerate(local if not fuse else []):
            agg.switch(k)
            mode = es.ES_STASH_BORROW if i == len(local) - 1 else es.ES_STASH_COPY
            if args.per_bucket:
                for b in range(B):
                    agg.stash(k, b, grads[k][b], mode)
            else:
                agg.stash_many(k, range(B), grads[k], mode)
        mark(1)
        if args.per_bucket:
            for b in range(B):
                agg.allreduce(b, outs[b])
        else:
            agg.allreduce_many(range(B), outs)
        mark(2)

    use_graph = not args.no_graph
    stream = torch.cuda.Stream(device=dev)
    for _ in range(2):
        with torch.cuda.stream(stream):
            step()
    torch.cuda.synchronize()
    graph = graph_prof = graph_phase = None
    marks = [torch.cuda.Event(enable_timing=True, external=use_graph) for _ in range(3)]
    if use_graph:
        # Three captures of the same step: without timing events (the K steps
        # we time), with phase-boundary events only (replayed once after the
        # timed region: stash and allreduce phases with every overlap intact),
        # and with per-kernel event nodes (replayed once after that: per-kind
        # durations).
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=stream):
            step()
        graph_phase = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph_phase, stream=stream):
            step(marks)
        agg.profile(True)
        agg.profile_reset()
        graph_prof = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph_prof, stream=stream):
            step()
        agg.profile(False)
        torch.cuda.synchronize()
        for _ in range(max(args.warmup, 3)):
            with torch.cuda.stream(stream):
                graph.replay()
        with torch.cuda.stream(stream):
            graph_prof.replay()
        torch.cuda.synchronize()
    else:
        for _ in range(max(args.warmup, 3)):
            with torch.cuda.stream(stream):
                step()
        torch.cuda.synchronize()
        agg.profile(True)
        agg.profile_reset()

    clocks = Clocks(local_rank)
    clocks.start()
    time.sleep(0.3)
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_start = time.time()
    with torch.cuda.stream(stream):
        for i in range(args.steps):
            if flush is not None:                 # L2 flush between timed steps (untimed): write 4x L2,
                flush.zero_()                     # then read it back so the flush's own dirty lines are
                flush_sink.copy_(flush_words.amax())   # drained here, not inside the next timed step
            starts[i].record(stream)
            if graph is not None:
                graph.replay()                    # the K timed steps carry no instrumentation
            else:
                step(marks if i == args.steps - 2 else None)
            ends[i].record(stream)
    torch.cuda.synchronize()
    t_end = time.time()
    if graph is not None:
        # after (outside) the timed region, in the same steady state (queued back to back behind
        # plain replays, no host sync in between): one replay with phase-boundary events, one with
        # per-kernel event pairs, each prepared like a timed step
        with torch.cuda.stream(stream):
            for g_ in (graph, graph, graph_phase, graph, graph_prof):
                if flush is not None:
                    flush.zero_()
                    flush_sink.copy_(flush_words.amax())
                g_.replay()
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop(t_start, t_end)
    step_ms = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    ms = sum(step_ms) / len(step_ms)
    ms = max_over_ranks(ms)

    kinds = {"stash": es.ES_KERNEL_STASH, "fold": es.ES_KERNEL_FOLD, "swap": es.ES_KERNEL_SWAP,
             "gather": es.ES_KERNEL_GATHER, "barrier": es.ES_KERNEL_BARRIER}
    prof = {k: agg.profile_query(v) for k, v in kinds.items()}   # (launches, ms, bytes)
    agg.profile(False)
    steps_profiled = 1 if graph is not None else args.steps
    launches_per_step = sum(p[0] for p in prof.values()) / (1 if graph is not None else args.steps)
    fl_n, fl_ms, fl_bytes = prof["fold"]
    payload = workloads.payload_bytes(name)
    value = payload / (ms / 1e3) / 1e9
    peak, peak_src = peaks()
    # Roofline of every HBM kernel of the step; `roofline` is the dominant one
    # (largest share of the profiled step's device time).
    traffic_all = {}
    tfile = os.path.join(ROOT, "profiles", f"traffic_{name}_g{G}.json")
    if os.path.exists(tfile) and not (args.incremental or args.per_bucket or args.no_fuse or args.no_graph
                                      or args.inplace):
        with open(tfile) as f:
            traffic_all = json.load(f)

    # Phase timing (fused G=1 step only, where the stash phase holds nothing but stash kernels with
    # their fused switches and the allreduce phase nothing but the fold): events at the phase
    # boundaries of one timed step, no event between kernels, so early start and PDL overlap stay
    # intact.  The per-kernel event pairs of the profiled step add ~1-5 us per launch.
    phase_ms = None
    if fuse and G == 1 and (graph is not None or args.steps >= 2):
        phase_ms = {"stash": marks[0].elapsed_time(marks[1]), "fold": marks[1].elapsed_time(marks[2])}

    def roof(kind, kname):
        n_, ms_, bytes_ = prof[kind]
        if n_ == 0 or ms_ <= 0:
            return None
        ev_us = ms_ / n_ * 1e3                                       # per-kernel event pairs
        if phase_ms is not None and kind in phase_ms:
            us, how = phase_ms[kind] * 1e3 / (n_ / steps_profiled), "phase events (no event between launches)"
        else:
            us, how = ev_us, "per-launch event pairs"
        a = bytes_ / n_ / (us / 1e6) / 1e9
        return {"bound": "hbm", "kernel": kname, "achieved": round(a, 1), "peak": peak, "unit": "GB/s",
                "frac": round(a / peak, 4), "traffic": traffic_all.get(f"{kname}_dram_bytes_per_launch"),
                "algorithmic_bytes_per_launch": int(bytes_ / n_), "launches_per_step": int(n_ / steps_profiled),
                "avg_launch_us": round(us, 2), "timing": how, "avg_launch_us_event_pairs": round(ev_us, 2),
                "share_of_step": round(us * n_ / steps_profiled / 1e3 / ms, 3), "peak_source": peak_src,
                "frac_of_nominal": round(a / HBM_NOMINAL_GBPS, 4)}

    roofs = {k: r for k, r in (("k_fold", roof("fold", "k_fold")), ("k_stash", roof("stash", "k_stash")),
                               ("k_gather", roof("gather", "k_gather"))) if r is not None}
    dominant = max(roofs.values(), key=lambda r: r["share_of_step"]) if roofs else None

    line = {
        "metric": METRIC, "value": round(value, 3), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms, 5), "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": cfg["dtype"], "data": "synthetic",
        "config": {**workload_config(args, cfg, G), "graph": graph is not None,
                   **({"rehearsal": "all ranks on cuda:0 (functional check of the N>1 path, not a scaling number)"}
                      if rehearse else {}),
                   "api": "per-bucket" if args.per_bucket else ("incremental" if args.incremental else
                                                               ("zero-copy-inplace" if args.inplace else
                                                                ("batched" if args.no_fuse else "batched+fused-switch")))
                   + (" +stash-background" if args.stash_background else "")
                   + (" +peer-push" if args.peer_push else ""),
                   "l2": ("inputs larger than L2 (%.1f MB of EST gradients per GPU per step)" % (in_bytes / 1e6))
                   if flush is None else "L2 flushed between timed steps (512 MB write, then read back: "
                                                  "no flush lines left dirty to drain inside the timed step)"},
        "roofline": dominant,
        "roofline_by_kernel": roofs,
        # the whole step against the same peak: every kernel's algorithmic bytes of one step divided by
        # the UNPROFILED step time (per-kernel event pairs above add ~1-5 us per launch; this has none)
        "step_roofline": {"achieved": round(sum(v[2] for v in prof.values()) / steps_profiled / (ms / 1e3) / 1e9, 1),
                          "peak": peak, "unit": "GB/s",
                          "frac": round(sum(v[2] for v in prof.values()) / steps_profiled / (ms / 1e3) / 1e9 / peak, 4),
                          "bytes_per_step": int(sum(v[2] for v in prof.values()) / steps_profiled),
                          "frac_of_nominal": round(sum(v[2] for v in prof.values()) / steps_profiled / (ms / 1e3) / 1e9
                                                   / HBM_NOMINAL_GBPS, 4)},
        "breakdown_ms_per_step": {k: round(v[1] / steps_profiled, 4) for k, v in prof.items()},
        "per_kernel": {k: {"launches_per_step": int(v[0] / steps_profiled),
                           "algorithmic_GBps": round(v[2] / (v[1] / 1e3) / 1e9, 1) if v[1] > 0 else None,
                           "us_per_launch": round(v[1] / max(v[0], 1) * 1e3, 2)} for k, v in prof.items()},
        # SURVEY 8(d)'s narrower metric: es_allreduce time only (stashes already done)
        "allreduce_only": {"ms": round(fl_ms / steps_profiled, 4),
                           "GBps": round(payload / (fl_ms / steps_profiled / 1e3) / 1e9, 1) if fl_ms > 0 else None},
        "gpu_launches": int(round(launches_per_step * args.steps)),
        "step_ms_p10_p50_p90": [round(float(np.percentile(step_ms, q)), 4) for q in (10, 50, 90)],
        "clocks": clk,
    }

    # ---- context-switch latency (reported separately) ----
    if len(local) > 1:
        n_sw = len(local) * max(1, 64 // len(local))      # a cycle: the graph ends on the EST it starts from
        seq = [local[(i + 1) % len(local)] for i in range(n_sw)]
        with torch.cuda.stream(stream):
            agg.switch(local[0])
        torch.cuda.synchronize()
        gsw = torch.cuda.CUDAGraph()
        with torch.cuda.graph(gsw, stream=stream):
            for k in seq:
                agg.switch(k)
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            for _ in range(3):
                gsw.replay()
            s0.record(stream)
            for _ in range(10):
                gsw.replay()
            s1.record(stream)
        torch.cuda.synchronize()
        us = s0.elapsed_time(s1) * 1e3 / (10 * n_sw)
        ctx_bytes = sum(snb)
        line["switch"] = {"us_per_switch": round(us, 3), "context_bytes": ctx_bytes,
                          "algorithmic_GBps": round(4 * ctx_bytes / (us / 1e6) / 1e9, 1),
                          "timed": f"{10 * n_sw} back-to-back es_switch_context in a CUDA graph",
                          "share_of_step": round(us * len(local) / 1e3 / ms, 4)}

    # ---- parity of the timed outputs against the oracle on sampled windows (+ cpu_baseline) ----
    if rank == 0:
        import oracle  # test infrastructure: the cpu_baseline leg and parity check only
        gen_cache = {}

        def fetch(k, b, s, n):
            if k in grads:
                t = grads[k][b][s:s + n]
            else:                                   # remote EST: regenerate its seeded input
                if (k, b) not in gen_cache:
                    gen_cache[(k, b)] = workloads.est_bucket(name, k, b, device=dev)
                t = gen_cache[(k, b)][s:s + n]
            t = t.cpu()
            return t.numpy() if t.dtype == torch.float32 else t.view(torch.int16).numpy().view(np.uint16)

        budget = args.cpu_seconds if (world == 1 and not args.no_cpu) else 1.0
        gbs, sample, windows = oracle_windows(name, fetch, budget)
        mism = 0
        checked = 0
        for b, s, n, want in windows:
            got = outs[b][s:s + n].cpu()
            got = got.numpy() if got.dtype == torch.float32 else got.view(torch.int16).numpy().view(np.uint16)
            w = want.view(np.uint32 if want.dtype == np.float32 else np.uint16)
            g_ = got.view(w.dtype)
            mism += int((w != g_).sum())
            checked += n
        line["parity"] = {"checked_elements": checked, "mismatched_words": mism, "vs": "CPU oracle, bit-exact"}
        # SURVEY 8(d) bit-exact flag: SHA-256 of the whole reduced bucket set (bucket order, raw
        # words).  Equal across G and mappings (D1); the scaling run's lines can be compared.
        h = hashlib.sha256()
        for o in outs:
            h.update(o.view(torch.uint8).cpu().numpy().tobytes())
        line["output_sha256"] = h.hexdigest()
        if payload <= 3e9:
            # the whole output against the oracle (seconds of single-thread C for these sizes)
            ho, mism_all = hashlib.sha256(), 0
            for b, (L_b, d_b) in enumerate(buckets):
                want = oracle.reduce([fetch(k, b, 0, L_b) for k in range(N)], d_b)
                ho.update(want.tobytes())
                got = outs[b].view(torch.uint8).cpu().numpy()
                mism_all += int((got.view(want.dtype) != want).sum()) if want.dtype != np.float32 else \
                    int((got.view(np.uint32) != want.view(np.uint32)).sum())
            line["parity"].update({"full_output_checked": True, "full_output_mismatched_words": mism_all,
                                   "oracle_sha256": ho.hexdigest(),
                                   "sha256_equal": ho.hexdigest() == line["output_sha256"]})
        if world == 1 and not args.no_cpu:
            line["cpu_baseline"] = {"value": round(gbs, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                                    "sample": sample, "host_cores_available": cores_used()}
            # the oracle also on all host cores (same code, one window per thread)
            gbs_mc, sample_mc = oracle_all_cores(name, fetch, cores_used())
            line["cpu_baseline_all_cores"] = {"value": round(gbs_mc, 4), "unit": "GB/s", "cores": cores_used(),
                                              "kind": "oracle", "sample": sample_mc}

    # ---- e2e: public API with host buffers (pinned H2D in, D2H out, inside the timed region) ----
    if not args.no_e2e:
        host = {k: [g.cpu().pin_memory() for g in grads[k]] for k in local}
        # two live-gradient buffers: EST i+1's H2D (copy stream) overlaps EST i's stash (compute stream)
        live_grad = [[torch.empty_like(grads[local[0]][b]) for b in range(B)] for _ in range(2)]
        host_out = [torch.empty(o.shape, dtype=o.dtype).pin_memory() for o in outs]
        h2d = len(local) * sum(n for n, _ in buckets) * esz
        d2h = sum(n for n, _ in buckets) * esz

        # The result's D2H runs on its own stream (PCIe is full duplex), overlapping the next step's H2D;
        # the next aggregation waits for it before overwriting `outs`.
        h2d_stream = torch.cuda.Stream(device=dev)
        d2h_stream = torch.cuda.Stream(device=dev)
        d2h_done = torch.cuda.Event()
        d2h_done.record(d2h_stream)
        free = [torch.cuda.Event(), torch.cuda.Event()]     # live buffer j may be overwritten
        for e in free:
            e.record(stream)
        landed = [torch.cuda.Event(), torch.cuda.Event()]   # live buffer j holds its EST's gradients
        ready = torch.cuda.Event()

        def e2e_step():
            # the same call sequence as the timed step (switch-in, fused stash + switch per EST, BORROW
            # for the last, one allreduce), each EST's gradients first landing from pinned host memory
            for i, k in enumerate(local):
                j = i % 2
                h2d_stream.wait_event(free[j])
                with torch.cuda.stream(h2d_stream):
                    for b in range(B):                 # "backward" lands in a live buffer
                        live_grad[j][b].copy_(host[k][b], non_blocking=True)
                landed[j].record(h2d_stream)
                stream.wait_event(landed[j])
                if i == 0:
                    agg.switch(k)
                if i == len(local) - 1:
                    agg.stash_many(k, range(B), live_grad[j], es.ES_STASH_BORROW)
                else:                                  # a COPY stash releases the buffer at once
                    agg.stash_and_switch(k, range(B), live_grad[j], local[i + 1], es.ES_STASH_COPY)
                    free[j].record(stream)
            stream.wait_event(d2h_done)
            agg.allreduce_many(range(B), outs)
            ready.record(stream)
            free[(len(local) - 1) % 2].record(stream)  # the BORROWed buffer is free after the allreduce
            d2h_stream.wait_event(ready)
            with torch.cuda.stream(d2h_stream):
                for b in range(B):
                    host_out[b].copy_(outs[b], non_blocking=True)
            d2h_done.record(d2h_stream)

        k_e2e = max(3, min(args.steps, 10))
        with torch.cuda.stream(stream):
            e2e_step()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(stream):
            e0.record(stream)
            for _ in range(k_e2e):
                e2e_step()
            stream.wait_event(d2h_done)                   # the last result is on the host
            stream.wait_event(free[0])
            stream.wait_event(free[1])
            e1.record(stream)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1) / k_e2e
        ems = max_over_ranks(ems)
        # The e2e ceiling: the step's H2D bytes over this host link, the link's rate measured as plain
        # pinned H2D copies of the step's input tensors, repeated to >= 256 MB so small steps are not
        # latency-bound (the D2H runs in the other direction, overlapped).
        flat = [t for k in local for t in host[k]]
        dst = [torch.empty_like(live_grad[0][b]) for b in range(B)]
        rounds = max(1, -(-(256 << 20) // h2d))
        h2d_ms = float("inf")
        for _ in range(6):                                # best of 5 after one warm-up pass
            c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(h2d_stream):
                c0.record(h2d_stream)
                for _r in range(rounds):
                    for i, t in enumerate(flat):
                        dst[i % B].copy_(t, non_blocking=True)
                c1.record(h2d_stream)
            torch.cuda.synchronize()
            if _ > 0:
                h2d_ms = min(h2d_ms, c0.elapsed_time(c1) / rounds)
        h2d_ms = max_over_ranks(h2d_ms)
        h2d_gbs = h2d / (h2d_ms / 1e3) / 1e9
        line["e2e"] = {"value": round(payload / (ems / 1e3) / 1e9, 3), "unit": "GB/s", "h2d_bytes_per_step": h2d,
                       "d2h_bytes_per_step": d2h, "ms_per_step": round(ems, 3), "steps": k_e2e,
                       "roofline": {"bound": "pcie_h2d", "peak": round(h2d_gbs, 2), "unit": "GB/s",
                                    "peak_source": "measured here: pinned H2D copies of the step's input tensors",
                                    "t_min_ms": round(h2d_ms, 3), "frac": round(h2d_ms / ems, 4)}}
    agg.sync()
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
