#!/bin/bash
# round-2 GPU batch 2: new NEXT-1 (G > 1) and tile-pipelined CHAIN tests first, the full GPU suite,
# the N > 1 rehearsals on the current bench (fixed open-failure hook, rehearsal-aware rooflines),
# the five G = 1 lines, and a steady-state (no cache control) ncu pass over the default command.
O=gpurun_out/r02b; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "incremental or chain_tile" > $O/pytest_new.log 2>&1; echo "rc $?" >> $O/pytest_new.log
timeout 600 python -m pytest tests/test_gpu_peer_graph.py -x -q -p no:cacheprovider > $O/pytest_graph.log 2>&1; echo "rc $?" >> $O/pytest_graph.log
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
# steady state: the default command's graph replays, no cache control (dirty L2 lines left by one
# kernel are written back under the next, as in the timed step); skip the 2 eager warm-up steps
timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  -k 'regex:k_(fold|stash)' -s 64 -c 96 --csv --log-file $O/steady_swin_b.csv python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-full-parity > $O/steady_swin_b.log 2>&1
timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  -k 'regex:k_(fold|stash)' -s 16 -c 24 --csv --log-file $O/steady_resnet50.csv python bench.py --config resnet50 --steps 3 --warmup 3 --no-cpu --no-e2e --no-full-parity > $O/steady_resnet50.log 2>&1
echo done3 >> $O/done.txt
