#!/bin/bash
# round-2 GPU batch 4: NVML NVLink counter support, MPS availability, and fresh ncu evidence of the
# round-2 build for the headline config (launch list + --set full of k_fold / k_stash).
O=gpurun_out/r02d; mkdir -p $O
python scripts/nvml_nvlink_probe.py > $O/nvml_probe.json 2> $O/nvml_probe.err
{ which nvidia-cuda-mps-control nvidia-cuda-mps-server; nvidia-smi -q | grep -i -A3 "compute mode"; } > $O/mps.txt 2>&1
nvidia-smi nvlink -gt d > $O/nvlink_gt.txt 2>&1
timeout 1800 bash scripts/ncu_configs.sh swin_b bert_base > $O/ncu_configs.log 2>&1
cp gpurun_out/launches_swin_b.csv gpurun_out/full_fold_swin_b.ncu-rep gpurun_out/full_stash_swin_b.ncu-rep $O/ 2>/dev/null
cp gpurun_out/launches_bert_base.csv gpurun_out/full_fold_bert_base.ncu-rep gpurun_out/full_stash_bert_base.ncu-rep $O/ 2>/dev/null
timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  -k 'regex:k_(fold|stash)' -s 24 -c 36 --csv --log-file $O/steady_bert_base.csv python bench.py --config bert_base --steps 3 --warmup 3 --no-cpu --no-e2e --no-full-parity --no-next1 > $O/steady_bert_base.log 2>&1
echo done > $O/done.txt
