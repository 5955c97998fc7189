#!/bin/bash
# Build libkcore variants with different compile-time knobs for tools/sweep.py.
set -e
cd "$(dirname "$0")/.."
NCCL_DIR=$(python -c "import nvidia.nccl,os;print(list(nvidia.nccl.__path__)[0])")
OUT=paper_conf_icde_ahmady0gcz23_b200/lib/variants
mkdir -p $OUT
build() {
  tag=$1; shift
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC \
    --expt-relaxed-constexpr -Iinclude -I$NCCL_DIR/include -shared "$@" \
    paper_conf_icde_ahmady0gcz23_b200/csrc/kcore.cu paper_conf_icde_ahmady0gcz23_b200/csrc/kcore_mg.cu paper_conf_icde_ahmady0gcz23_b200/csrc/kcore_extract.cu paper_conf_icde_ahmady0gcz23_b200/csrc/kcore_mpm.cu paper_conf_icde_ahmady0gcz23_b200/csrc/kcore_testhooks.cu paper_conf_icde_ahmady0gcz23_b200/csrc/kcore_mgd.cu \
    -o $OUT/$tag.so -L$NCCL_DIR/lib -l:libnccl.so.2 -Xlinker -rpath=$NCCL_DIR/lib
  echo built $tag
}
while read -r tag flags; do
  [ -z "$tag" ] && continue
  build $tag $flags &
  while [ $(jobs -r | wc -l) -ge 6 ]; do sleep 1; done
done < "${1:-tools/variants.txt}"
wait
