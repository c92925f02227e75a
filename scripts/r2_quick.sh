#!/bin/bash
# quick: stream tests + bench line + optional ncu of the protected stream kernel
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/ncu
timeout 900 python -m pytest tests/test_gpu_stream.py -x -q 2>&1 | tail -5 > gpurun_out/stream_tests.log
timeout 300 python bench.py --no-cpu-baseline --steps 200 ${BENCH_ARGS} > gpurun_out/bench_quick.log 2>&1
python -c "import json; L=[l for l in open('gpurun_out/bench_quick.log') if l.startswith('{')]; d=json.loads(L[-1]); print('bench', d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct'], d['config']['c_format'])" > gpurun_out/bench_quick.txt 2>&1
if [ -n "$NCU" ]; then
KREGEX="k_stream<\(bool\)1, \(bool\)0" W=7pt128 TAG=stream_prot SKIP=3 bash scripts/ncu_one.sh
KREGEX="k_stream<\(bool\)0, \(bool\)0" W=7pt128 TAG=stream_plain SKIP=3 bash scripts/ncu_one.sh
fi
cat gpurun_out/stream_tests.log gpurun_out/bench_quick.txt
