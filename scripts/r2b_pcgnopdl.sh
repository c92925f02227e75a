#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
rm -f gpurun_out/pn.log
for rep in 1 2; do
  ABFT_NO_PDL=1 timeout 300 python scripts/pcg_time.py | sed 's/^/nopdl_all /' >> gpurun_out/pn.log 2>&1
  timeout 300 python scripts/pcg_time.py | sed 's/^/default /' >> gpurun_out/pn.log 2>&1
done
cat gpurun_out/pn.log
