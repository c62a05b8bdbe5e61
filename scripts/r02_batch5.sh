#!/bin/bash
# round-2 GPU batch 5: the GPU suite with whole-output full-size parity, NEXT-1 at full size and in
# training, then a 500-seed fuzz of schedules / maps / layouts / options (pipelined CHAIN, NEXT-1).
O=gpurun_out/r02e; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "full_size" > $O/pytest_full_size.log 2>&1; echo "rc $?" >> $O/pytest_full_size.log
timeout 600 python -m pytest tests/test_gpu_training_d1.py -x -q -p no:cacheprovider > $O/pytest_training.log 2>&1; echo "rc $?" >> $O/pytest_training.log
timeout 2100 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc $?" >> $O/pytest_gpu.log
ES_FUZZ_SEEDS=500 timeout 1800 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k random_schedules > $O/fuzz_500.log 2>&1; echo "rc $?" >> $O/fuzz_500.log
echo done > $O/done.txt
