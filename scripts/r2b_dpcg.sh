#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parallel.py -q -x > gpurun_out/dpcg_tests.log 2>&1; echo "rc=$?" >> gpurun_out/dpcg_tests.log
ABFT_DIST_PCG_EAGER=1 timeout 600 python bench.py --pcg-dist --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/pcg_dist_eager.log 2>&1
timeout 600 python bench.py --pcg-dist --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/pcg_dist_graph.log 2>&1
timeout 600 python bench.py --strong --workload 27pt256 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/strong_27pt256.log 2>&1
tail -2 gpurun_out/dpcg_tests.log
for f in gpurun_out/pcg_dist_eager.log gpurun_out/pcg_dist_graph.log; do python -c "
import json,sys
d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1])
print(sys.argv[1], {k:(v['ms'],v['iters']) for k,v in d['results'].items()})" $f; done
tail -c 700 gpurun_out/strong_27pt256.log
