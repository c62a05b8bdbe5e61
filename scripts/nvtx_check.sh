#!/bin/bash
# NVTX ranges of the C-ABI calls (SURVEY 5 tracing), checked with ncu's NVTX filter on one GPU:
# inside "es_allreduce_many" ranges only k_fold launches, inside "es_stash_and_switch" only
# k_stash launches.  Writes gpurun_out/nvtx_{allreduce,stash}.csv; summarise with
#   python scripts/ncu_summary.py launches gpurun_out/nvtx_allreduce.csv
mkdir -p gpurun_out
B="python bench.py --config tiny --no-graph --steps 3 --warmup 3 --no-e2e --no-cpu"
for r in allreduce_many:allreduce stash_and_switch:stash; do
  range=${r%%:*}; tag=${r##*:}
  timeout 300 ncu --nvtx --nvtx-include "es_${range}/" --metrics gpu__time_duration.sum --clock-control none \
      --csv --log-file gpurun_out/nvtx_$tag.csv $B > gpurun_out/nvtx_$tag.log 2>&1
done
