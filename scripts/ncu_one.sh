#!/bin/bash
# one ncu --set full capture: KREGEX (demangled name regex), W (workload), TAG
cd $GRAFT_REPO_ROOT; O=gpurun_out/ncu; mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k "regex:${KREGEX}" -s ${SKIP:-2} -c 1 -o $O/${TAG} -f python bench.py --workload ${W} --steps 3 --warmup 3 --no-cpu-baseline > $O/${TAG}.log 2>&1
tail -2 $O/${TAG}.log
