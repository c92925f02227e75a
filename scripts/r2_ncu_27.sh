#!/bin/bash
# k_stream protected vs plain on 27pt256 (configs[3] single GPU)
cd $GRAFT_REPO_ROOT; O=gpurun_out/ncu; mkdir -p $O
timeout 600 python bench.py --workload 27pt256 --no-cpu-baseline --steps 20 > $O/b27.jsonl 2>&1
KREGEX="k_stream<\(bool\)1, \(bool\)0" W=27pt256 TAG=s27p SKIP=3 bash scripts/ncu_one.sh
KREGEX="k_stream<\(bool\)0, \(bool\)0" W=27pt256 TAG=s27q SKIP=3 bash scripts/ncu_one.sh
for T in s27p s27q; do
  python scripts/ncu_summary.py $O/$T.ncu-rep 524288 30 > $O/${T}_summary.txt 2>&1
  python scripts/ncu_sass_stalls.py $O/$T.ncu-rep 524288 60 > $O/${T}_sass.txt 2>&1
  rm -f $O/$T.ncu-rep
done
