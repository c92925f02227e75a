#!/bin/bash
# R-MAT scale 24: launch list + one full ncu capture of k_hub and k_irr<CHECK>
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/ncu
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/ncu/launches_rmat24.csv python bench.py --workload rmat24 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu/rmat24_launch.log 2>&1
KREGEX="k_hub" W=rmat24 TAG=rmat24_hub SKIP=2 bash scripts/ncu_one.sh
KREGEX="k_irr<\(bool\)1, \(bool\)0" W=rmat24 TAG=rmat24_irr SKIP=2 bash scripts/ncu_one.sh
for t in rmat24_hub rmat24_irr; do
  python scripts/ncu_summary.py gpurun_out/ncu/$t.ncu-rep 1 40 > gpurun_out/ncu/$t.summary.txt 2>&1
  python scripts/ncu_sass_stalls.py gpurun_out/ncu/$t.ncu-rep 1 30 > gpurun_out/ncu/$t.stalls.txt 2>&1
  python scripts/ncu_lines.py gpurun_out/ncu/$t.ncu-rep 1 40 > gpurun_out/ncu/$t.lines.txt 2>&1
  rm -f gpurun_out/ncu/$t.ncu-rep
done
du -sh gpurun_out
