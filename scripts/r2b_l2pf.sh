#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_stream.py -q -x > gpurun_out/pf_tests.log 2>&1; echo "rc=$?" >> gpurun_out/pf_tests.log
rm -f gpurun_out/pf.log
for rep in 1 2; do for P in 1 0; do for w in 7pt128 7pt192 27pt256 27pt128; do
  echo -n "nopf=$P $w: " >> gpurun_out/pf.log
  if [ $P = 1 ]; then E="ABFT_STREAM_NO_L2PF=1"; else E="ABFT_X=0"; fi
  env $E timeout 300 python bench.py --no-cpu-baseline --steps 100 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/pf.log 2>&1
done; done; done
tail -2 gpurun_out/pf_tests.log; cat gpurun_out/pf.log
