#!/bin/bash
# R-MAT path profile: launch list + one ncu --set full capture of k_general<CHECK>
cd $GRAFT_REPO_ROOT; O=gpurun_out/rmat; mkdir -p $O
W=${W:-rmat20}
timeout 600 python bench.py --workload $W --no-cpu-baseline --steps 100 > $O/bench_$W.jsonl 2> $O/bench_$W.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
  --log-file $O/launches_$W.csv python bench.py --workload $W --steps 5 --warmup 3 --no-cpu-baseline > $O/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:k_general<.bool.1' -s 2 -c 1 -o $O/k_general_$W -f python bench.py --workload $W --steps 3 --warmup 3 --no-cpu-baseline > $O/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k 'regex:k_lean<.bool.1' -s 2 -c 1 -o $O/k_lean_$W -f python bench.py --workload $W --steps 3 --warmup 3 --no-cpu-baseline > $O/ncu_full2.log 2>&1
tail -3 $O/*.log; cat $O/bench_$W.jsonl | head -c 600
