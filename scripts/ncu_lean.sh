#!/bin/bash
# one ncu --set full capture of k_lean<CHECK> on the bench workload
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_lean -s 12 -c 1 -o gpurun_out/prof_lean python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log
