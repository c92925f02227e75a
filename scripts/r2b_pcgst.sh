#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
timeout 900 python -m pytest tests -m gpu -q -x -k "pcg" > gpurun_out/pcgst_tests.log 2>&1; echo "rc=$?" >> gpurun_out/pcgst_tests.log
for lib in libabft_before.so libabft.so libabft_before.so libabft.so; do
  ABFT_LIB=$PWD/$P/$lib timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline --pcg-seeds 1 --pcg-reps 3 > gpurun_out/pcgst_$lib.jsonl 2>/dev/null
  python -c "
import json,sys
d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1])
print(sys.argv[1], {k:(v['ms'],v['iters']) for k,v in d['results'].items() if k.endswith('lam0')})" gpurun_out/pcgst_$lib.jsonl >> gpurun_out/pcgst.log
done
tail -2 gpurun_out/pcgst_tests.log; cat gpurun_out/pcgst.log
