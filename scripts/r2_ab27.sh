#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_stream.py -x -q 2>&1 | tail -2 > gpurun_out/ab27_tests.log
LIBS="libabft.so" WORKLOADS="27pt128 27pt256 7pt128" bash scripts/sweep_libs.sh > gpurun_out/ab27.log 2>&1
