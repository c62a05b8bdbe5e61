#!/bin/bash
# ncu evidence for every G = 1 bench config (SURVEY 8(d) "ncu on one representative
# k_fold / k_stash launch per config").  One GPU; run under gpurun:
#   bash scripts/ncu_configs.sh [configs...]       (default: all five)
# Writes, per config c, into gpurun_out/:
#   launches_<c>.csv    ncu --metrics gpu__time_duration.sum launch list of `bench.py --no-graph`
#                       (our kernels only; cold cache, serialised: compare shares, not absolutes)
#   full_fold_<c>.ncu-rep, full_stash_<c>.ncu-rep
#                       ncu --set full of one k_fold / one k_stash launch after the warm-up
# Summarise here with scripts/ncu_summary.py (launches | full | traffic).
mkdir -p gpurun_out
CONFIGS=${*:-"tiny resnet50 vgg19 bert_base swin_b"}
B="python bench.py --no-graph --no-e2e --no-cpu --steps 3 --warmup 3"
for c in $CONFIGS; do
  # launches per step: (n_local - 1) fused stash+switch launches + 1 fold; x 6 steps
  case $c in tiny) n=4;; resnet50) n=8;; vgg19) n=16;; bert_base) n=12;; swin_b) n=32;; esac
  cnt=$((6 * (n + 1)))
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:k_(fold|stash|swap)' \
      -c $cnt --csv --log-file gpurun_out/launches_$c.csv $B --config $c > gpurun_out/launches_$c.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fold -s 2 -c 1 -f \
      -o gpurun_out/full_fold_$c $B --config $c > gpurun_out/full_fold_$c.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_stash -s $((2 * (n - 1))) -c 1 -f \
      -o gpurun_out/full_stash_$c $B --config $c > gpurun_out/full_stash_$c.log 2>&1
  echo "$c done: $(ls gpurun_out/*_$c* | tr '\n' ' ')"
done
# The default bench command itself (CUDA graph, PDL, early-start stashes) for the default workload:
# the first 2 eager warm-up steps + the graph replays after them, 9 of our launches per ResNet-50 step.
if [[ " $CONFIGS " == *" resnet50 "* ]]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:k_(fold|stash|swap)' \
      -c 90 --csv --log-file gpurun_out/launches_resnet50_default_cmd.csv python bench.py --steps 5 --warmup 3 \
      > gpurun_out/launches_resnet50_default_cmd.log 2>&1
fi
