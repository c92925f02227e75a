#!/bin/bash
# k_stream protected vs plain on 7pt128: instruction mix per group, stalls, SASS hot lines
cd $GRAFT_REPO_ROOT; O=gpurun_out/ncu; mkdir -p $O
KREGEX="k_stream<\(bool\)1, \(bool\)0" W=7pt128 TAG=sp SKIP=3 bash scripts/ncu_one.sh
KREGEX="k_stream<\(bool\)0, \(bool\)0" W=7pt128 TAG=sq SKIP=3 bash scripts/ncu_one.sh
for T in sp sq; do
  python scripts/ncu_summary.py $O/$T.ncu-rep 65536 30 > $O/${T}_summary.txt 2>&1
  python scripts/ncu_sass_stalls.py $O/$T.ncu-rep 65536 80 > $O/${T}_sass.txt 2>&1
  ncu -i $O/$T.ncu-rep --page source --csv --print-source=sass > $O/${T}_source.csv 2>/dev/null
  rm -f $O/$T.ncu-rep
done
