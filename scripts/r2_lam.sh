#!/bin/bash
# Item 5: overhead vs lambda (resident plans) on configs[1] and PCG configs[4]
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stream.py -q -x > gpurun_out/lam_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/lam_tests.log
timeout 600 python bench.py --lam-sweep --workload 7pt128 --steps 200 --warmup 10 > gpurun_out/lam_7pt128.jsonl 2> gpurun_out/lam_7pt128.err
[ "$PCG" = 1 ] && timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/lam_pcg.jsonl 2> gpurun_out/lam_pcg.err
tail -3 gpurun_out/lam_tests.log
