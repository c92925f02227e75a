#!/bin/bash
# compare alternative builds of libabft (ABFT_LIB) on the bench workload
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; rm -f gpurun_out/sweep_libs.log
for lib in ${LIBS:-libabft.so}; do
  for w in ${WORKLOADS:-7pt128}; do
  echo -n "$lib $w: " >> gpurun_out/sweep_libs.log
  ABFT_LIB=$PWD/paper_conf_dsn_schollbkw16_b200/$lib timeout 300 python bench.py --no-cpu-baseline --steps 300 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/sweep_libs.log 2>&1
  done
done
cat gpurun_out/sweep_libs.log
