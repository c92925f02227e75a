#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
rm -f gpurun_out/upd.log
for lib in libabft.so libabft_upd4.so libabft.so libabft_upd4.so; do
  ABFT_LIB=$PWD/$P/$lib timeout 300 python scripts/pcg_time.py >> gpurun_out/upd.log 2>&1
done
ABFT_LIB=$PWD/$P/libabft_upd4.so timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k pcg >> gpurun_out/upd.log 2>&1
cat gpurun_out/upd.log | tail -8
