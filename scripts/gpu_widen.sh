#!/bin/bash
# SURVEY §8(f)1-2 measurements: dense-check comparison, coverage / F1 (ours vs
# dense check, and per b_s), overhead per b_s.
cd $GRAFT_REPO_ROOT; O=gpurun_out/widen; mkdir -p $O
for w in 7pt128 27pt128 rmat20 5pt64; do
  timeout 600 python bench.py --compare --workload $w --steps 100 > $O/compare_$w.jsonl 2> $O/compare_$w.err
done
timeout 1500 python scripts/coverage.py > $O/coverage.jsonl 2> $O/coverage.err
for w in 7pt128 27pt128; do for bs in 1 2 4 8 16 32; do
  timeout 600 python bench.py --workload $w --block-size $bs --no-cpu-baseline --steps 50 >> $O/bs_sweep_$w.jsonl 2>> $O/bs_sweep.err
done; done
tail -3 $O/*.err | head -30
