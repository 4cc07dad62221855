#!/bin/bash
# Build libsat from the working tree with sat_kernel.cuh replaced by $1, into
# paper_conf_cluster_chenwttm18_b200/libsat_<$2>.so (same-box A/B experiments).
set -e
KFILE=$(realpath "$1"); NAME=$2
ROOT=$(cd "$(dirname "$0")/.." && pwd)
TMP=$(mktemp -d)
mkdir -p $TMP/include $TMP/pkg/csrc
cp $ROOT/paper_conf_cluster_chenwttm18_b200/csrc/* $TMP/pkg/csrc/
cp $KFILE $TMP/pkg/csrc/sat_kernel.cuh
cp $ROOT/include/libsat.h $TMP/include/
NCCL_INC=$(python -c "import nvidia.nccl,os;print(os.path.join(list(nvidia.nccl.__path__)[0],'include'))")
cd $TMP/pkg/csrc
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC -shared \
  --expt-relaxed-constexpr -I $NCCL_INC "${@:3}" -o $ROOT/paper_conf_cluster_chenwttm18_b200/libsat_$NAME.so \
  sat_runtime.cu sat_host.cu sat_dist.cu sat_query.cu $( [ -f sat_brlt.cu ] && echo sat_brlt.cu ) -ldl
rm -rf $TMP
echo built libsat_$NAME.so
