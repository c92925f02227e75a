#!/bin/bash
# k_stream ring-shape sweep on the bench workload (env switches, same box)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; : > gpurun_out/sweep_stream.log
while read -r line; do
  [ -z "$line" ] && continue
  echo -n "$line: " >> gpurun_out/sweep_stream.log
  env $line timeout 300 python bench.py --no-cpu-baseline --steps 300 --workload ${W:-7pt128} 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['ft_overhead_pct']))" >> gpurun_out/sweep_stream.log 2>&1
done < ${CFGS:-scripts/r2_sweep_cfgs.txt}
cat gpurun_out/sweep_stream.log
