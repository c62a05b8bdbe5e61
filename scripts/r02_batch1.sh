#!/bin/bash
# round-2 GPU batch 1: GPU tests, default bench (swin_b), rehearsals (G=2/4/8) incl. the fallback hook
O=gpurun_out/r02a; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc $?" >> $O/pytest_gpu.log
timeout 600 python bench.py > $O/bench_default.json 2> $O/bench_default.err
R() { n=$1; out=$2; shift; shift; timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node=$n --master-addr 127.0.0.1 --master-port $((29500+RANDOM%1000)) bench.py --gpus $n --rehearse-same-gpu --no-cpu --steps 5 --warmup 3 "$@" > $O/$out.json 2> $O/$out.err; }
R 2 reh_resnet50_g2 --config resnet50
R 4 reh_resnet50_g4 --config resnet50
R 8 reh_resnet50_g8 --config resnet50
R 8 reh_bert_g8rr --config bert_base --mapping round_robin
R 2 reh_swin_g2 --config swin_b
R 2 reh_resnet50_g2_failopen --config resnet50 --simulate-peer-failure open
R 2 reh_resnet50_g2_failparity --config resnet50 --simulate-peer-failure parity
echo done1 > $O/done.txt
# launch list of the default command (swin_b), cold-cache serialised per-launch times
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file $O/launches_swin_b_default.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-full-parity > $O/ncu_launch.log 2>&1
echo done2 >> $O/done.txt
