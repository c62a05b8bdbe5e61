#!/bin/bash
# round-2 GPU batch 12: the N > 1 rehearsals under CUDA MPS (ranks run concurrently, each on
# 100/G % of the SMs) -- fine-grained cross-process interleavings of the peer protocols.
rm -rf gpurun_out/mps
bash scripts/rehearse_mps.sh 2 resnet50 --steps 20
bash scripts/rehearse_mps.sh 4 resnet50 --steps 20
bash scripts/rehearse_mps.sh 8 resnet50 --steps 20
bash scripts/rehearse_mps.sh 8 bert_base --mapping round_robin --steps 20
bash scripts/rehearse_mps.sh 2 swin_b --steps 20
bash scripts/rehearse_mps.sh 4 swin_b --steps 20
bash scripts/rehearse_mps.sh 8 vgg19 --steps 20
TAG=_inc bash scripts/rehearse_mps.sh 4 resnet50 --incremental --steps 20
TAG=_failparity bash scripts/rehearse_mps.sh 2 resnet50 --simulate-peer-failure parity --steps 20
echo done > gpurun_out/mps/done.txt
