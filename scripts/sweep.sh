#!/bin/bash
# tuning sweep of k_lean: carveout x stages x warps (bench numbers only)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
run() { timeout 300 python bench.py --no-cpu-baseline --steps 300 ${BENCH_ARGS} 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms']))"; }
for cv in ${CARVES:-100 75}; do for st in ${STAGES:-2}; do for w in ${WARPS:-4 2}; do
  echo -n "carve=$cv stages=$st warps=$w: " >> gpurun_out/sweep.log
  ABFT_CARVEOUT=$cv ABFT_STAGES=$st ABFT_WARPS=$w run >> gpurun_out/sweep.log 2>&1
done; done; done
cat gpurun_out/sweep.log
