#!/bin/bash
# round-2 GPU batch 18: final build -- GPU suite, compute-sanitizer, the five G = 1 lines, smoke.
O=gpurun_out/r02q; mkdir -p $O
timeout 2100 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc $?" >> $O/pytest_gpu.log
for c in swin_b resnet50 tiny vgg19 bert_base; do
  timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err
done
timeout 1800 bash scripts/sanitize_all.sh > $O/sanitize.log 2>&1; cp gpurun_out/sanitizer.txt $O/
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
echo done > $O/done.txt
