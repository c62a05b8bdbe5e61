#!/bin/bash
# Fold variants, same box, interleaved (build each with scripts/build_fold_variant.sh first):
#   v0 = round-2 fold (opening contribution loaded alone, then batches of 8);
#   v1 = opening contribution inside the first batch (fp32 and bf16);
#   v2 = v1 + __launch_bounds__(256, 4);
#   v3 = v0 for fp32, v2 for bf16 (k_fold_b) -- the kept design.
# VARIANTS / CONFIGS / REPS override the sets.
# Each variant's libes is copied over the package's libes.so for its runs (bits must not change:
# every line carries sampled oracle parity and output_sha256).
O=${OUT:-gpurun_out/fold_variants}; mkdir -p $O
P=paper_conf_sc_lixyszrljlllq23_b200
cp $P/libes.so $O/libes_current.so
for rep in ${REPS:-1 2}; do
  for v in ${VARIANTS:-v0 v1 v2}; do
    cp $P/variants/libes_$v.so $P/libes.so
    for c in ${CONFIGS:-resnet50 bert_base swin_b tiny vgg19}; do
      timeout 300 python bench.py --config $c --no-cpu --no-e2e --no-next1 --no-full-parity > $O/${v}_${c}_$rep.json 2> $O/${v}_${c}_$rep.err
    done
  done
done
cp $O/libes_current.so $P/libes.so
echo done > $O/done.txt
