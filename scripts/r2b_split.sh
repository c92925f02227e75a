#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
timeout 900 python -m pytest tests -m gpu -q -x -k "pcg or cg1 or dist or parallel" > gpurun_out/sp_tests.log 2>&1; echo "rc=$?" >> gpurun_out/sp_tests.log
rm -f gpurun_out/sp.log
for rep in 1 2; do for lib in libabft_nosplit.so libabft.so; do
  ABFT_LIB=$PWD/$P/$lib timeout 300 python scripts/pcg_time.py >> gpurun_out/sp.log 2>&1
done; done
tail -2 gpurun_out/sp_tests.log; cat gpurun_out/sp.log
