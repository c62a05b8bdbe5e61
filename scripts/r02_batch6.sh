#!/bin/bash
# round-2 GPU batch 6: the kept fold (v3: fp32 as before, bf16 merged first batch + 64-register
# bound) against v0, then the parity tests that exercise every fold instantiation.
O=gpurun_out/r02f; mkdir -p $O
OUT=gpurun_out/fold_variants2 VARIANTS="v0 v3" CONFIGS="bert_base swin_b resnet50 vgg19 tiny" REPS="1 2" bash scripts/fold_variant_probe.sh
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_switch.py tests/test_gpu_knobs.py tests/test_gpu_peer_graph.py -q -p no:cacheprovider -x -k "not full_size" > $O/pytest_parity.log 2>&1; echo "rc $?" >> $O/pytest_parity.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc $?" >> $O/smoke.log
echo done > $O/done.txt
