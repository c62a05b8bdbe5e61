#!/bin/bash
# N>1 bench rehearsal with every rank on one GPU under CUDA MPS: the ranks' kernels run
# concurrently (each client limited to 100/G % of the SMs) instead of time-slicing the GPU, so the
# peer protocols (device barriers, per-tile flags over CUDA IPC) see fine-grained cross-process
# interleavings.  Still not a G-GPU number (one HBM, one SM pool).
#   bash scripts/rehearse_mps.sh G config [bench args...]
G=${1:?G}; C=${2:?config}; shift; shift
O=gpurun_out/mps; mkdir -p $O
export CUDA_MPS_PIPE_DIRECTORY=/tmp/mps_pipe CUDA_MPS_LOG_DIRECTORY=/tmp/mps_log
mkdir -p $CUDA_MPS_PIPE_DIRECTORY $CUDA_MPS_LOG_DIRECTORY
nvidia-cuda-mps-control -d || { echo "mps: no daemon" > $O/mps_${C}_g$G.err; exit 0; }
export CUDA_MPS_ACTIVE_THREAD_PERCENTAGE=$((100 / G)) ES_BARRIER_TIMEOUT_S=30
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node=$G --master-addr 127.0.0.1 \
  --master-port $((29600 + RANDOM % 300)) bench.py --gpus $G --rehearse-same-gpu --no-cpu --steps 5 --warmup 3 \
  --config $C "$@" > $O/mps_${C}_g$G$TAG.json 2> $O/mps_${C}_g$G$TAG.err
echo "rc $?" >> $O/mps_${C}_g$G$TAG.err
echo quit | nvidia-cuda-mps-control
cp /tmp/mps_log/control.log $O/mps_control_${C}_g$G.log 2>/dev/null
