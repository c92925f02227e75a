#!/bin/bash
# One profiling round on the GPU box; outputs under gpurun_out/prof_round/.
# Summarised into profiles/ by scripts/summarize_round.py (run locally).
cd $GRAFT_REPO_ROOT; O=gpurun_out/prof_round; mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.max.sm,clocks.max.mem --format=csv > $O/gpu.csv
timeout 600 python bench.py > $O/bench.jsonl 2> $O/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference.jsonl 2>&1
# launch list of the bench command (cold-cache, serialised: compare shares)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file $O/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $O/ncu_launch.log 2>&1
# full capture of the fused kernel (protected) and of the plain kernel
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lean -s 12 -c 1 \
  -o $O/k_lean -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $O/ncu_full.log 2>&1
timeout 900 python bench.py --pcg > $O/pcg.jsonl 2>&1
timeout 900 python scripts/coverage.py > $O/coverage.jsonl 2>&1
ls -la $O
