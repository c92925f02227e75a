#!/bin/bash
# GPU round: parity tests, smoke, bench (+ optional tuning sweep and ncu).
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py --cpu-seconds 5 > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
if [ -n "$SWEEP" ]; then
  for st in 2 3 4; do for w in 2 4; do
    echo "stages=$st warps=$w" >> gpurun_out/sweep.log
    ABFT_STAGES=$st ABFT_WARPS=$w timeout 300 python bench.py --no-cpu-baseline --steps 300 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith(\"{\")]; d=json.loads(L[-1]); print(d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct'])" >> gpurun_out/sweep.log 2>&1
  done; done
fi
if [ -n "$NCU" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lean -s 12 -c 2 -o gpurun_out/prof_fused python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
fi
tail -5 gpurun_out/pytest_gpu.log; tail -3 gpurun_out/smoke.log; tail -2 gpurun_out/bench.log; cat gpurun_out/sweep.log 2>/dev/null
