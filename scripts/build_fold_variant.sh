#!/bin/bash
# Builds paper_conf_sc_lixyszrljlllq23_b200/variants/libes_<tag>.so from csrc/kernels.cu at git
# revision <rev> (default: the working tree) and every other current source, with the same nvcc
# flags as _build.py plus any extra -D flags, for scripts/fold_variant_probe.sh.
#   bash scripts/build_fold_variant.sh v0 c52d3db
#   bash scripts/build_fold_variant.sh v3
set -e
tag=${1:?tag}; rev=${2:-}; shift; shift || true
C=paper_conf_sc_lixyszrljlllq23_b200/csrc
T=$(mktemp -d); cp $C/*.h $T/
if [ -n "$rev" ]; then git show $rev:$C/kernels.cu > $T/kernels.cu; else cp $C/kernels.cu $T/; fi
NCCL_INC=$(python -c "import nvidia.nccl, os; print(os.path.join(list(nvidia.nccl.__path__)[0], 'include'))")
mkdir -p paper_conf_sc_lixyszrljlllq23_b200/variants
nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -ftz=false -prec-div=true -prec-sqrt=true \
  -fmad=false -Xcompiler -fPIC,-Wall,-ffp-contract=off -shared -I $NCCL_INC -I include -I $C "$@" \
  -o paper_conf_sc_lixyszrljlllq23_b200/variants/libes_$tag.so \
  $C/api_allreduce.cpp $C/api_core.cpp $C/api_peer_context.cpp $C/api_stash.cpp $C/plan.cpp \
  $C/transport_loopback.cpp $C/transport_nccl.cpp $T/kernels.cu -ldl -lpthread
echo built variants/libes_$tag.so
