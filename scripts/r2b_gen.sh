#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
rm -f gpurun_out/gen.log
for rep in 1 2; do for lib in libabft.so libabft_g6.so; do for w in rmat24 rmat20; do
  echo -n "$lib $w: " >> gpurun_out/gen.log
  ABFT_LIB=$PWD/$P/$lib timeout 300 python bench.py --no-cpu-baseline --steps 30 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/gen.log 2>&1
done; done; done
cat gpurun_out/gen.log
