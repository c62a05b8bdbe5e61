#!/bin/bash
# Run-to-run spread of the G = 1 bench lines: each config R times (fresh process each time).
#   bash scripts/bench_repeat.sh [R] [configs...]  -> gpurun_out/repeat_<config>.jsonl
mkdir -p gpurun_out
R=${1:-3}; shift
for c in ${*:-resnet50 vgg19 bert_base swin_b tiny}; do
  : > gpurun_out/repeat_$c.jsonl
  for i in $(seq 1 $R); do
    timeout 600 python bench.py --config $c --no-e2e --cpu-seconds 1 2>/dev/null | tail -1 >> gpurun_out/repeat_$c.jsonl
  done
done
