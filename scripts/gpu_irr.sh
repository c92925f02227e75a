#!/bin/bash
# k_irr bring-up: GPU parity tests, R-MAT / stencil bench lines, launch list
cd $GRAFT_REPO_ROOT; O=gpurun_out/irr; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
for w in rmat20 7pt128 ${EXTRA}; do
  timeout 900 python bench.py --workload $w --no-cpu-baseline --steps 100 > $O/bench_$w.jsonl 2> $O/bench_$w.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
  --log-file $O/launches_rmat20.csv python bench.py --workload rmat20 --steps 5 --warmup 3 --no-cpu-baseline > $O/ncu_launch.log 2>&1
tail -4 $O/pytest_gpu.log
for f in $O/bench_*.jsonl; do python -c "import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['ms_per_step'], d['plain_ms'], d['ft_overhead_pct'], d['roofline']['frac'], d['config'].get('general_groups'))"; done
