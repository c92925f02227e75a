#!/bin/bash
# round 2: stream kernel parity + bench A/B
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_stream.py -x -q 2>&1 | tail -30 > gpurun_out/stream_tests.log
timeout 300 python bench.py --no-cpu-baseline --steps 200 > gpurun_out/bench_stream.log 2>&1
ABFT_NO_POS=1 timeout 300 python bench.py --no-cpu-baseline --steps 200 > gpurun_out/bench_nopos.log 2>&1
for f in bench_stream bench_nopos; do python -c "import json; L=[l for l in open('gpurun_out/$f.log') if l.startswith('{')]; d=json.loads(L[-1]); print('$f', d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct'], d['config']['c_format'])" ; done
