#!/bin/bash
# NVLink bytes of a multi-GPU bench run (for a box with G >= 2 GPUs; not runnable on one GPU).
#   bash scripts/nvlink_bytes.sh G [bench args...]
# Reads nvidia-smi's per-link data-throughput counters (KiB, tx/rx) on every GPU before and after
# `torchrun --nproc-per-node G bench.py --gpus G ...` and prints the per-GPU deltas. No ncu replay:
# ncu on a multi-rank command would replay the peer-barrier kernels and hang. Compare the delta
# per step with profiles/r01_plan_roofline.md's NVLink bytes (the whole run also holds warm-up,
# the switch-latency graph and the e2e leg: use --no-e2e and subtract a --steps 0 run if needed).
# For kernel-level counts on ONE rank of a single-process loopback run: ncu metrics
# nvlrx__bytes_data_user / nvltx__bytes_data_user (names queried on this pool's B200,
# profiles/r01_nvlink_env.md).
G=${1:?G}; shift
snap() { nvidia-smi nvlink -gt d 2>/dev/null; }
snap > gpurun_out/nvlink_before.txt
python -m torch.distributed.run --nnodes=1 --nproc-per-node $G --master-addr 127.0.0.1 --master-port 29533 \
    bench.py --gpus $G "$@" > gpurun_out/nvlink_bench_g$G.jsonl
snap > gpurun_out/nvlink_after.txt
python - <<'PY'
import re
def parse(p):
    d, gpu = {}, None
    for line in open(p):
        m = re.match(r"GPU (\d+):", line)
        if m:
            gpu = int(m.group(1)); continue
        m = re.search(r"Link (\d+): Data (Tx|Rx): (\d+) KiB", line)
        if m and gpu is not None:
            d[(gpu, m.group(2))] = d.get((gpu, m.group(2)), 0) + int(m.group(3))
    return d
a, b = parse("gpurun_out/nvlink_before.txt"), parse("gpurun_out/nvlink_after.txt")
for k in sorted(b):
    print(f"GPU {k[0]} {k[1]}: {(b[k] - a.get(k, 0)) * 1024 / 1e6:.1f} MB")
PY
