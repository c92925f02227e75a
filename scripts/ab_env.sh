#!/bin/bash
# A/B of environment switches on the bench workloads: ENVS="A=1 B=2 -" (- = none)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; rm -f gpurun_out/ab_env.log
for e in ${ENVS:--}; do for w in ${WORKLOADS:-7pt128}; do
  echo -n "$e $w: " >> gpurun_out/ab_env.log
  if [ "$e" = "-" ]; then E=""; else E="$e"; fi
  env $E timeout 300 python bench.py --no-cpu-baseline --steps 200 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/ab_env.log 2>&1
done; done
cat gpurun_out/ab_env.log
