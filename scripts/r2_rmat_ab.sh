#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; : > gpurun_out/rmat_ab.log
for cfg in "ABFT_X=1" "ABFT_HUB_SAME_STREAM=1" "ABFT_LIB=$PWD/paper_conf_dsn_schollbkw16_b200/libabft_u8.so"; do
  for w in rmat24 rmat20; do
  echo -n "$cfg $w: " >> gpurun_out/rmat_ab.log
  env $cfg timeout 600 python bench.py --no-cpu-baseline --steps 30 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['ft_overhead_pct'], d['cusparse_plain'].get('ms_per_step')))" >> gpurun_out/rmat_ab.log 2>&1
  done
done
cat gpurun_out/rmat_ab.log
