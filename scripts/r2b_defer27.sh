#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_stream.py -q -x > gpurun_out/d27_tests.log 2>&1; echo "rc=$?" >> gpurun_out/d27_tests.log
rm -f gpurun_out/d27.log
for rep in 1 2; do for D in 0 1; do for w in 27pt128 27pt256; do
  echo -n "defer=$D $w: " >> gpurun_out/d27.log
  ABFT_STREAM_DEFER=$D timeout 300 python bench.py --no-cpu-baseline --steps 100 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/d27.log 2>&1
done; done; done
tail -2 gpurun_out/d27_tests.log; cat gpurun_out/d27.log
