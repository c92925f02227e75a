#!/bin/bash
# full GPU suite + lambda sweep
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/full_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/full_tests.log
timeout 600 python bench.py --lam-sweep --workload 7pt128 --steps 200 --warmup 10 > gpurun_out/lam_7pt128.jsonl 2> gpurun_out/lam_7pt128.err
[ "$PCG" = 1 ] && timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/lam_pcg.jsonl 2> gpurun_out/lam_pcg.err
tail -3 gpurun_out/full_tests.log
