#!/bin/bash
# A/B: libs x env settings on the bench workload(s), interleaved repeats
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; rm -f gpurun_out/ab_env.log
for rep in 1 2; do
for lib in ${LIBS:-libabft.so}; do
  for envs in ${ENVS:-NONE=1}; do
  for w in ${WORKLOADS:-7pt128}; do
  echo -n "$lib $envs $w: " >> gpurun_out/ab_env.log
  env $envs ABFT_LIB=$PWD/paper_conf_dsn_schollbkw16_b200/$lib timeout 300 python bench.py --no-cpu-baseline --steps 300 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/ab_env.log 2>&1
  done; done; done; done
cat gpurun_out/ab_env.log
