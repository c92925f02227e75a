#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/ncu
timeout 900 python -m pytest tests/test_gpu_stream.py -x -q 2>&1 | tail -5 > gpurun_out/stream_tests.log
KREGEX="k_stream<\(bool\)1, \(bool\)0" W=7pt128 TAG=stream_prot SKIP=3 bash scripts/ncu_one.sh
KREGEX="k_stream<\(bool\)0, \(bool\)0" W=7pt128 TAG=stream_plain SKIP=3 bash scripts/ncu_one.sh
