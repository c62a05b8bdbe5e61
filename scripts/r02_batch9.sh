#!/bin/bash
# round-2 GPU batch 9: the five G = 1 lines on the final build, then the run-to-run spread (3 fresh
# processes per config, --no-e2e --cpu-seconds 1).
O=gpurun_out/r02i; mkdir -p $O
for c in swin_b resnet50 tiny vgg19 bert_base; do
  timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err
done
echo done1 > $O/done.txt
bash scripts/bench_repeat.sh 3
mkdir -p $O/repeat; cp gpurun_out/repeat_*.jsonl $O/repeat/
echo done2 >> $O/done.txt
