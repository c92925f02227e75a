#!/bin/bash
# One profiling round on the GPU box; outputs under gpurun_out/prof_round/.
# Summarised into profiles/ by scripts/summarize_round.py (run locally).
cd $GRAFT_REPO_ROOT; O=gpurun_out/prof_round; mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.max.sm,clocks.max.mem --format=csv > $O/gpu.csv
timeout 600 python bench.py > $O/bench.jsonl 2> $O/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference.jsonl 2>&1
for w in 27pt128 27pt256 rmat20 rmat24 5pt64; do
  timeout 600 python bench.py --workload $w --no-cpu-baseline --steps 100 > $O/bench_$w.jsonl 2>&1
done
# launch list of the bench command (cold-cache, serialised: compare shares)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file $O/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $O/ncu_launch.log 2>&1
# full capture of the fused kernel (protected)
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:k_lean<.bool.1, .bool.0, .int.1, .int.2, .bool.1, .bool.0, .bool.0>' -s 4 -c 1 \
  -o $O/k_lean -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $O/ncu_full.log 2>&1
timeout 900 python bench.py --pcg > $O/pcg.jsonl 2>&1
timeout 900 python scripts/coverage.py > $O/coverage.jsonl 2>&1
for w in 7pt128 27pt128 rmat20 5pt64; do
  timeout 600 python bench.py --compare --workload $w --steps 100 > $O/compare_$w.jsonl 2>&1
done
ls -la $O
