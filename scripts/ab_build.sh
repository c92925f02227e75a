#!/bin/bash
# Build libabft_base.so from a git revision (default HEAD) for same-box A/B
# timing against the working tree's libabft.so (scripts/sweep_libs.sh).
set -e
cd "$(dirname "$0")/.."
REV=${1:-HEAD}
T=$(mktemp -d)
git archive $REV paper_conf_dsn_schollbkw16_b200/csrc include | tar -x -C $T
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 \
  -Xcompiler -ffp-contract=off -fmad=false -Xcompiler -fPIC -shared -cudart static $(python -c "from paper_conf_dsn_schollbkw16_b200 import _build as b; print(' '.join(b.nccl_flags()))") \
  -o paper_conf_dsn_schollbkw16_b200/libabft_base.so $T/paper_conf_dsn_schollbkw16_b200/csrc/abft.cu
rm -rf $T
