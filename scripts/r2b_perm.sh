#!/bin/bash
# popularity-ordered x: parity + R-MAT A/B
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/ncu
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "popularity or irregular or rmat or hub or bench_workloads" > gpurun_out/perm_tests.log 2>&1; echo "rc=$?" >> gpurun_out/perm_tests.log
for W in rmat24 rmat22 rmat20; do
  for P in 0 1; do ABFT_COLPERM=$P timeout 400 python bench.py --no-cpu-baseline --steps 30 --workload $W > gpurun_out/perm_${W}_$P.log 2>&1; done
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_rmat24.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --workload rmat24 > gpurun_out/ncu_launch_rmat.log 2>&1
KREGEX="k_hub" W=rmat24 TAG=hub24 SKIP=3 bash scripts/ncu_one.sh
KREGEX="k_irr<\(bool\)1" W=rmat24 TAG=irr24 SKIP=3 bash scripts/ncu_one.sh
tail -3 gpurun_out/perm_tests.log
for f in gpurun_out/perm_rmat*.log; do echo "== $f"; python - "$f" <<'PY'
import json,sys
L=[l for l in open(sys.argv[1]) if l.startswith('{')]
if L:
    d=json.loads(L[-1]); print(d['ms_per_step'], d['plain_ms'], d['ft_overhead_pct'], d['roofline']['frac'], d['config'].get('col_perm'))
PY
done
