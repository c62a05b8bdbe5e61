#!/usr/bin/env python
"""Launch-shape probe for small steps (development tool, not a bench line).

The tiny config (N=4, one 1M-element fp32 bucket, 16.8 MB per step) is bound
by kernel latency, not HBM.  This captures bench.py's fused G=1 step as a CUDA
graph under several es_set_launch_override shapes (applied to stash and fold)
and times graph replays with an L2 flush (write + read back) between steps.
Bits never depend on the shape (tests/test_gpu_parity.py); the probe checks
that every shape's output equals the default shape's.

  python scripts/tiny_latency_probe.py [--config tiny] [--steps 200]
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
    ap.add_argument("--config", default="tiny")
    ap.add_argument("--steps", type=int, default=200)
    a = ap.parse_args()
    import torch
    from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads
    from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    cfg = workloads.config(a.config)
    N, buckets = cfg["N"], cfg["buckets"]
    B = len(buckets)
    snb = workloads.state_nbytes()
    agg = Aggregator(N, 1, 0, [0] * N, buckets, state_nbytes=snb, device=dev)
    live = [torch.zeros(n, dtype=torch.uint8, device=dev) for n in snb]
    agg.register_state(live)
    for k in range(N):
        for i, blob in enumerate(workloads.est_state(a.config, k)):
            agg.init_state(k, i, blob)
    grads = [[workloads.est_bucket(a.config, k, b, device=dev) for b in range(B)] for k in range(N)]
    outs = [agg.new_out(b) for b in range(B)]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    fw = flush.view(torch.int32)
    sink = torch.zeros((), dtype=torch.int32, device=dev)
    stream = torch.cuda.Stream(device=dev)

    def step():
        agg.switch(0)
        for k in range(N):
            if k == N - 1:
                agg.stash_many(k, range(B), grads[k], es.ES_STASH_BORROW)
            else:
                agg.stash_and_switch(k, range(B), grads[k], k + 1, es.ES_STASH_COPY)
        agg.allreduce_many(range(B), outs)

    ref = None
    shapes = [(0, 0), (148, 256), (296, 256), (444, 256), (592, 256), (888, 256), (1184, 256), (296, 128),
              (592, 128), (1184, 128), (2368, 128)]
    for blocks, threads in shapes:
        agg.set_launch_override(blocks, threads)
        with torch.cuda.stream(stream):
            step()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=stream):
            step()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
        with torch.cuda.stream(stream):
            for _ in range(5):
                g.replay()
            for s, e in ev:
                flush.zero_()
                sink.copy_(fw.amax())
                s.record(stream)
                g.replay()
                e.record(stream)
        torch.cuda.synchronize()
        ms = [s.elapsed_time(e) for s, e in ev]
        out = torch.cat([o.view(torch.uint8) for o in outs]).cpu()
        if ref is None:
            ref = out
        print(json.dumps({"blocks": blocks, "threads": threads, "median_us": round(1e3 * statistics.median(ms), 2),
                          "p10_us": round(1e3 * sorted(ms)[len(ms) // 10], 2), "bits_equal_default": bool(torch.equal(out, ref))}),
              flush=True)
    agg.set_launch_override(0, 0)
    agg.close()


if __name__ == "__main__":
    main()
