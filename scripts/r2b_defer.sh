#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
timeout 900 python -m pytest tests/test_gpu_stream.py tests/test_gpu_parity.py tests/test_gpu_dense.py -q -x > gpurun_out/defer_tests.log 2>&1; echo "rc=$?" >> gpurun_out/defer_tests.log
rm -f gpurun_out/defer.log
for rep in 1 2; do for lib in libabft.so libabft_nodefer.so; do for w in 7pt128 7pt192 27pt256; do
  echo -n "$lib $w: " >> gpurun_out/defer.log
  ABFT_LIB=$PWD/$P/$lib timeout 300 python bench.py --no-cpu-baseline --steps 200 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/defer.log 2>&1
done; done; done
ABFT_LIB=$PWD/$P/libabft_e8.so python scripts/phase_probe.py 128 >> gpurun_out/defer.log 2>&1
tail -2 gpurun_out/defer_tests.log; cat gpurun_out/defer.log
