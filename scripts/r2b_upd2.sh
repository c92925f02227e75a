#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
rm -f gpurun_out/upd2.log
for rep in 1 2; do for lib in libabft.so libabft_p4.so libabft_u5.so libabft_p4u5.so; do
  ABFT_LIB=$PWD/$P/$lib timeout 300 python scripts/pcg_time.py >> gpurun_out/upd2.log 2>&1
done; done
cat gpurun_out/upd2.log
