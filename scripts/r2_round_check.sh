#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CFGS=scripts/r2_cfgs_27.txt W=27pt128 bash scripts/r2_sweep_stream.sh > /dev/null 2>&1; cp gpurun_out/sweep_stream.log gpurun_out/sweep27_128.log
timeout 300 python bench.py --no-cpu-baseline --steps 100 --workload 27pt256 > gpurun_out/bench_27pt256.log 2>&1
timeout 300 python bench.py --no-cpu-baseline --steps 200 > gpurun_out/bench_7pt.log 2>&1
bash scripts/r2_sanitize.sh
cat gpurun_out/sweep27_128.log; tail -c 700 gpurun_out/bench_27pt256.log; tail -c 400 gpurun_out/bench_7pt.log
