#!/bin/bash
# One GPU: the five G = 1 bench lines into gpurun_out/bench_<config>.json (copy the last line of
# each to profiles/r01_bench_<config>_g1.json after checking clocks and parity).
mkdir -p gpurun_out
for c in ${*:-resnet50 tiny vgg19 bert_base swin_b}; do
  timeout 600 python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
  echo "$c exit $?"
done
