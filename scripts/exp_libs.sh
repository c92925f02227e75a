#!/bin/bash
# Build timing-experiment variants of libabft.so (-DABFT_EXP=n, see
# kernels_spmv.cuh) here on CPU; run with LIBS="..." scripts/sweep_libs.sh.
cd "$(dirname "$0")/.."
P=paper_conf_dsn_schollbkw16_b200
for e in ${EXPS:-1 2 3 4 5}; do
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 \
    -Xcompiler -ffp-contract=off -fmad=false -Xcompiler -fPIC -shared -cudart static $(python -c "from paper_conf_dsn_schollbkw16_b200 import _build as b; print(' '.join(b.nccl_flags()))") \
    -DABFT_EXP=$e -o $P/libabft_e$e.so $P/csrc/abft.cu &
done
wait
ls -la $P/libabft_e*.so
