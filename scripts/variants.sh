#!/bin/bash
# Build libabft_<name>.so variants with extra -D flags for same-box A/B runs:
#   scripts/variants.sh name1 "-DFOO=1" name2 "-DBAR=1 -DBAZ=2" ...
cd "$(dirname "$0")/.."
P=paper_conf_dsn_schollbkw16_b200
while [ $# -ge 2 ]; do
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 \
    -Xcompiler -ffp-contract=off -fmad=false -Xcompiler -fPIC -shared -cudart static $(python -c "from paper_conf_dsn_schollbkw16_b200 import _build as b; print(' '.join(b.nccl_flags()))") \
    $2 -o $P/libabft_$1.so $P/csrc/abft.cu &
  shift 2
done
wait
