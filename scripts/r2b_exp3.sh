#!/bin/bash
# where the protected k_stream time goes: EXP6 (no x gathers), EXP7 (no C pass)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
rm -f gpurun_out/exp3.log
for lib in libabft.so libabft_e6.so libabft_e7.so libabft.so; do
  for w in 7pt128 7pt192; do
    echo -n "$lib $w: " >> gpurun_out/exp3.log
    ABFT_LIB=$PWD/$P/$lib timeout 300 python bench.py --no-cpu-baseline --steps 300 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/exp3.log 2>&1
  done
done
cat gpurun_out/exp3.log
