#!/bin/bash
# round-2 cost decomposition of k_lean on 7pt128: EXP variants + ncu of the plain kernel
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2_gpu.csv
LIBS="libabft.so libabft_e1.so libabft_e2.so libabft_e3.so libabft_e5.so libabft.so" bash scripts/sweep_libs.sh
KREGEX="k_lean<false" W=7pt128 TAG=plain SKIP=3 bash scripts/ncu_one.sh
python scripts/ncu_summary.py gpurun_out/ncu/plain.ncu-rep 65536 30 > gpurun_out/ncu/plain_summary.txt 2>&1
