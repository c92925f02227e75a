#!/bin/bash
# b_s sweep 1..512 on the round-2 kernels
cd $GRAFT_REPO_ROOT; O=gpurun_out/bs2; mkdir -p $O
for w in 7pt128 27pt128; do for bs in 1 2 4 8 16 32 64 128 256 512; do
  timeout 600 python bench.py --workload $w --block-size $bs --no-cpu-baseline --steps 30 --warmup 3 2>> $O/bs_sweep.err | grep '^{' >> $O/bs_sweep_$w.jsonl
done; done
for w in 7pt128 27pt128; do python -c "
import json,sys
for l in open(sys.argv[1]):
    d=json.loads(l); print(sys.argv[1].split('_')[-1], d['config']['block_size'], d['ms_per_step'], d['plain_ms'], d['ft_overhead_pct'], d['roofline']['kernel'][:40])" $O/bs_sweep_$w.jsonl; done
