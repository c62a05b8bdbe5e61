#!/bin/bash
# round-2 GPU batch 20: both rehearsal sets on the final build (time-sliced processes; CUDA MPS).
O=gpurun_out/r02s; mkdir -p $O
R() { n=$1; out=$2; shift; shift; timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node=$n --master-addr 127.0.0.1 --master-port $((29500+RANDOM%1000)) bench.py --gpus $n --rehearse-same-gpu --no-cpu --steps 5 --warmup 3 "$@" > $O/$out.json 2> $O/$out.err; }
R 2 reh_resnet50_g2 --config resnet50
R 4 reh_resnet50_g4 --config resnet50
R 8 reh_resnet50_g8 --config resnet50
R 8 reh_bert_g8rr --config bert_base --mapping round_robin
R 2 reh_swin_g2 --config swin_b
R 2 reh_resnet50_g2_failopen --config resnet50 --simulate-peer-failure open
R 2 reh_resnet50_g2_failparity --config resnet50 --simulate-peer-failure parity
R 2 reh_resnet50_g2_incremental --config resnet50 --incremental
bash scripts/r02_batch12.sh
echo done > $O/done.txt
