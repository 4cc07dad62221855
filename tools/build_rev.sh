#!/bin/bash
# Build libsat from a git revision into paper_conf_cluster_chenwttm18_b200/libsat_<name>.so
# (same-box A/B timing: SAT_LIBRARY=<that .so> python tools/quick.py).
set -e
REV=$1; NAME=$2
ROOT=$(cd "$(dirname "$0")/.." && pwd)
TMP=$(mktemp -d)
mkdir -p $TMP/include $TMP/pkg/csrc
SRCS=""
for f in sat_kernel.cuh sat_runtime.cu sat_host.cu sat_dist.cu sat_query.cu sat_brlt.cu sat_internal.h; do
  if git -C $ROOT cat-file -e $REV:paper_conf_cluster_chenwttm18_b200/csrc/$f 2>/dev/null; then
    git -C $ROOT show $REV:paper_conf_cluster_chenwttm18_b200/csrc/$f > $TMP/pkg/csrc/$f
    case $f in *.cu) SRCS="$SRCS $f";; esac
  fi
done
git -C $ROOT show $REV:include/libsat.h > $TMP/include/libsat.h
NCCL_INC=$(python -c "import nvidia.nccl,os;print(os.path.join(list(nvidia.nccl.__path__)[0],'include'))")
cd $TMP/pkg/csrc
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC -shared \
  --expt-relaxed-constexpr -I $NCCL_INC "${@:3}" -o $ROOT/paper_conf_cluster_chenwttm18_b200/libsat_$NAME.so \
  $SRCS -ldl
rm -rf $TMP
echo built $ROOT/paper_conf_cluster_chenwttm18_b200/libsat_$NAME.so
