#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "pcg or cg1" > gpurun_out/pp_tests.log 2>&1; echo "rc=$?" >> gpurun_out/pp_tests.log
rm -f gpurun_out/pp.log
for rep in 1 2; do
  ABFT_PCG_NO_PDL=1 timeout 300 python scripts/pcg_time.py | sed 's/^/nopdl /' >> gpurun_out/pp.log 2>&1
  timeout 300 python scripts/pcg_time.py | sed 's/^/pdl /' >> gpurun_out/pp.log 2>&1
done
tail -2 gpurun_out/pp_tests.log; cat gpurun_out/pp.log
