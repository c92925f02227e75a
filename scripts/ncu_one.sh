#!/bin/bash
# one ncu --set full capture: KREGEX (demangled name regex), W (workload), TAG;
# UNITS (work units per launch, for per-unit instruction counts).  The report
# is summarised on the box and deleted unless KEEP=1 (reports are ~33 MB and
# gpurun copies back at most 64 MiB).
cd $GRAFT_REPO_ROOT; O=gpurun_out/ncu; mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k "regex:${KREGEX}" -s ${SKIP:-2} -c 1 -o $O/${TAG} -f python bench.py --workload ${W} --steps 3 --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > $O/${TAG}.log 2>&1
python scripts/ncu_summary.py $O/${TAG}.ncu-rep ${UNITS:-1} 30 > $O/${TAG}_summary.txt 2>&1
python scripts/ncu_lines.py $O/${TAG}.ncu-rep ${UNITS:-1} 40 >> $O/${TAG}_summary.txt 2>&1
[ "$KEEP" = 1 ] || rm -f $O/${TAG}.ncu-rep
tail -2 $O/${TAG}.log
