#!/bin/bash
# round-2 GPU batch 3: the GPU suite after the per-bucket chain partials fix, the N > 1 rehearsals
# and the five G = 1 lines on the current bench (NEXT-1 leg, phase_step_ms), compute-sanitizer.
O=gpurun_out/r02c; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "chain_tile or multi_step_reuse or compat_variants_loopback" > $O/pytest_chain.log 2>&1; echo "rc $?" >> $O/pytest_chain.log
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc $?" >> $O/pytest_gpu.log
R() { n=$1; out=$2; shift; shift; timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node=$n --master-addr 127.0.0.1 --master-port $((29500+RANDOM%1000)) bench.py --gpus $n --rehearse-same-gpu --no-cpu --steps 5 --warmup 3 "$@" > $O/$out.json 2> $O/$out.err; }
R 2 reh_resnet50_g2 --config resnet50
R 4 reh_resnet50_g4 --config resnet50
R 8 reh_resnet50_g8 --config resnet50
R 8 reh_bert_g8rr --config bert_base --mapping round_robin
R 2 reh_swin_g2 --config swin_b
R 2 reh_resnet50_g2_failopen --config resnet50 --simulate-peer-failure open
R 2 reh_resnet50_g2_failparity --config resnet50 --simulate-peer-failure parity
R 2 reh_resnet50_g2_incremental --config resnet50 --incremental
echo done1 > $O/done.txt
for c in swin_b resnet50 tiny vgg19 bert_base; do
  timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err
done
echo done2 >> $O/done.txt
timeout 2400 bash scripts/sanitize_all.sh > $O/sanitize.log 2>&1
cp gpurun_out/sanitizer.txt $O/sanitizer.txt 2>/dev/null
echo done3 >> $O/done.txt
