mkdir -p gpurun_out
R() { n=$1; shift; timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node=$n --master-addr 127.0.0.1 --master-port $((29500+RANDOM%1000)) bench.py --gpus $n --rehearse-same-gpu --no-cpu --steps 5 --warmup 3 "$@"; }
R 2 --config resnet50 --sched peer_auto > gpurun_out/reh_resnet50_g2.json 2> gpurun_out/reh.err
R 4 --config resnet50 --sched peer_chain > gpurun_out/reh_resnet50_g4.json 2>> gpurun_out/reh.err
R 8 --config resnet50 --sched peer --mapping random > gpurun_out/reh_resnet50_g8.json 2>> gpurun_out/reh.err
R 8 --config bert_base --sched peer_auto --mapping round_robin > gpurun_out/reh_bert_g8rr.json 2>> gpurun_out/reh.err
R 8 --config bert_base --sched peer_chain > gpurun_out/reh_bert_g8c.json 2>> gpurun_out/reh.err
R 8 --config resnet50 --sched peer --peer-push > gpurun_out/reh_resnet50_g8_push.json 2>> gpurun_out/reh.err
R 8 --config bert_base --sched peer --peer-push --mapping round_robin > gpurun_out/reh_bert_g8rr_push.json 2>> gpurun_out/reh.err
tail -5 gpurun_out/reh.err
