#!/bin/bash
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/inj_launches.csv python scripts/inj_probe.py 1e-8 > gpurun_out/inj_probe.log 2>&1
python scripts/launch_summary.py gpurun_out/inj_launches.csv > gpurun_out/inj_summary.txt 2>&1
