#!/bin/bash
# ncu --set full of the PCG vector kernels (192^3, fault-free probe)
O=gpurun_out/ncu; mkdir -p $O
for K in k_pcg_update k_pcg_p k_pcg_dotg; do
  timeout 900 ncu --set full --clock-control none --import-source on -k "regex:${K}\$" -s 20 -c 1 -o $O/pv_$K -f \
    python scripts/pcg_probe.py 0 0 > $O/pv_$K.log 2>&1
  python scripts/ncu_summary.py $O/pv_$K.ncu-rep 1 > $O/pv_${K}_summary.txt 2>&1
  python scripts/ncu_sass_stalls.py $O/pv_$K.ncu-rep > $O/pv_${K}_stalls.txt 2>&1
  rm -f $O/pv_$K.ncu-rep
done
