#!/bin/bash
# quick perf iteration: bench (no CPU baseline) + one ncu capture of k_lean<CHECK>
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python bench.py --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/bench_perf.log 2>&1
python -c "import json; L=[l for l in open('gpurun_out/bench_perf.log') if l.startswith('{')]; d=json.loads(L[-1]); print('value',d['value'],'ms',d['ms_per_step'],'plain_ms',d['plain_ms'],'fused_ms',d['roofline']['launch_ms'],'frac',d['roofline']['frac'],'ovh',d['ft_overhead_pct'])"
if [ -z "$NO_NCU" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lean -s 12 -c 1 -o gpurun_out/prof_lean -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/ncu_full.log 2>&1
fi
