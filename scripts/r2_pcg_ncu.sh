#!/bin/bash
mkdir -p gpurun_out
python scripts/pcg_probe.py 1e-8 7 > gpurun_out/pcgp_7.log 2>&1
python scripts/pcg_probe.py 1e-8 0 > gpurun_out/pcgp_0.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/pcgp_7.csv python scripts/pcg_probe.py 1e-8 7 > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/pcgp_0.csv python scripts/pcg_probe.py 1e-8 0 > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/pcgp_7.csv > gpurun_out/pcgp_7_summary.txt
python scripts/launch_summary.py gpurun_out/pcgp_0.csv > gpurun_out/pcgp_0_summary.txt
rm -f gpurun_out/pcgp_*.csv
