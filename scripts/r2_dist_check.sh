#!/bin/bash
# multi-GPU ABI on one GPU: parallel tests, strong-scaling line at N=1, sharded PCG at N=1
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parallel.py -x -q 2>&1 | tail -25 > gpurun_out/dist_tests.log
timeout 600 python bench.py --strong --workload 27pt256 --steps 20 --warmup 3 > gpurun_out/bench_strong1.log 2>&1
timeout 600 python bench.py --strong --workload 7pt128 --steps 50 --warmup 3 > gpurun_out/bench_strong7.log 2>&1
timeout 900 python bench.py --pcg-dist --pcg-reps 2 > gpurun_out/bench_pcgdist1.log 2>&1
tail -3 gpurun_out/dist_tests.log; tail -c 1500 gpurun_out/bench_strong1.log; tail -c 600 gpurun_out/bench_strong7.log; tail -c 2500 gpurun_out/bench_pcgdist1.log
