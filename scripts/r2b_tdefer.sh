#!/bin/bash
# DEFER as a template parameter + warp-cooperative hub chunk sums
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_stream.py tests/test_gpu_parity.py -q -x > gpurun_out/td_tests.log 2>&1; echo "rc=$?" >> gpurun_out/td_tests.log
rm -f gpurun_out/td.log
for rep in 1 2; do for w in 7pt128 7pt192 rmat24 rmat22; do
  echo -n "$w: " >> gpurun_out/td.log
  timeout 300 python bench.py --no-cpu-baseline --steps 100 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/td.log 2>&1
done; done
tail -2 gpurun_out/td_tests.log; cat gpurun_out/td.log
