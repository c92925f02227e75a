#!/bin/bash
# b_s sweep 1..512: overhead per b_s on 7pt128 / 27pt128, F1 per b_s
cd $GRAFT_REPO_ROOT; O=gpurun_out/bs; mkdir -p $O
for w in 7pt128 27pt128; do for bs in 1 2 4 8 16 32 64 128 256 512; do
  timeout 600 python bench.py --workload $w --block-size $bs --no-cpu-baseline --steps 30 --warmup 3 >> $O/bs_sweep_$w.jsonl 2>> $O/bs_sweep.err
done; done
timeout 900 python scripts/coverage.py --only bs --bs-runs 3000 > $O/coverage_bs.jsonl 2> $O/coverage_bs.err
tail -3 $O/*.err
