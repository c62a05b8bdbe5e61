"""Kernel launch-shape sweep on the GPU (development tool, not a bench line).

Times k_stash and k_fold of one workload under es_set_launch_override
(blocks, threads) with CUDA events, next to torch's copy_ as the copy
reference, and prints one JSON line per shape.  Results never change with
the shape (tests/test_gpu_parity.py::test_launch_config_invariance).
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads  # noqa: E402
from paper_conf_sc_lixyszrljlllq23_b200.aggregator import Aggregator  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="resnet50")
    ap.add_argument("--reps", type=int, default=20)
    a = ap.parse_args()
    cfg = workloads.config(a.config)
    N, buckets = cfg["N"], cfg["buckets"]
    B = len(buckets)
    agg = Aggregator(N, 1, 0, [0] * N, buckets)
    grads = [[workloads.est_bucket(a.config, k, b, device="cuda") for b in range(B)] for k in range(N)]
    outs = [agg.new_out(b) for b in range(B)]
    esz = 2 if cfg["dtype"] == "bf16" else 4
    tot = sum(n for n, _ in buckets)

    # torch copy reference over the same bytes as one EST's stash
    dst = [torch.empty_like(g) for g in grads[0]]
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for _ in range(3):
        for b in range(B):
            dst[b].copy_(grads[1][b])
    e0.record()
    for r in range(a.reps):
        for b in range(B):
            dst[b].copy_(grads[r % N][b])
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.reps
    print(json.dumps({"what": "torch_copy", "ms_per_est": round(ms, 4), "GBps": round(2 * tot * esz / ms / 1e6, 1)}))

    shapes = [(0, 0), (592, 256), (1184, 256), (2368, 256), (4736, 256), (9472, 256), (18944, 256), (37888, 256),
              (9472, 128), (18944, 128), (37888, 128), (37888, 64)]
    for blocks, threads in shapes:
        agg.set_launch_override(blocks, threads)
        for _ in range(2):
            for k in range(N):
                agg.stash_many(k, range(B), grads[k])
            agg.allreduce_many(range(B), outs)
        torch.cuda.synchronize()
        agg.profile(True)
        agg.profile_reset()
        for _ in range(a.reps):
            for k in range(N):
                agg.stash_many(k, range(B), grads[k])
            agg.allreduce_many(range(B), outs)
        torch.cuda.synchronize()
        st = agg.profile_query(es.ES_KERNEL_STASH)
        fo = agg.profile_query(es.ES_KERNEL_FOLD)
        agg.profile(False)
        print(json.dumps({"blocks": blocks, "threads": threads,
                          "stash_GBps": round(st[2] / st[1] / 1e6, 1), "stash_us_per_launch": round(st[1] / st[0] * 1e3, 2),
                          "fold_GBps": round(fo[2] / fo[1] / 1e6, 1), "fold_us_per_launch": round(fo[1] / fo[0] * 1e3, 2)}))
    agg.close()


if __name__ == "__main__":
    main()
