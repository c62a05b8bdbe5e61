#!/bin/bash
# round-2 GPU batch 7: final evidence on the current build (GPU suite, N > 1 rehearsals, five G = 1 lines).
O=gpurun_out/r02g; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1

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


echo done3 >> $O/done.txt
