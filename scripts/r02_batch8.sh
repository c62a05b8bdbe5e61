#!/bin/bash
# round-2 GPU batch 8: the five G = 1 lines with the e2e roofline's link rate from 64 MB copies.
O=gpurun_out/r02h; mkdir -p $O
for c in swin_b resnet50 tiny vgg19 bert_base; do
  timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err
done
echo done > $O/done.txt
