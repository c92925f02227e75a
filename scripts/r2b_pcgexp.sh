#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
rm -f gpurun_out/pcgexp.log
for lib in libabft.so libabft_e9.so libabft.so libabft_e9.so; do
  ABFT_LIB=$PWD/$P/$lib timeout 300 python scripts/pcg_time.py >> gpurun_out/pcgexp.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_pcg.csv python scripts/pcg_profile.py 192 1 > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/launches_pcg.csv > gpurun_out/launches_pcg_summary.txt
cat gpurun_out/pcgexp.log; head -12 gpurun_out/launches_pcg_summary.txt
