#!/bin/bash
# PCG checks: parity tests, default bench line, PCG time-to-solution
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "pcg or stream" > gpurun_out/pcg_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/pcg_tests.log
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/pcg_bench7.jsonl 2> gpurun_out/pcg_bench7.err
timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline --pcg-seeds ${SEEDS:-1} > gpurun_out/pcg_bench.jsonl 2> gpurun_out/pcg_bench.err
ABFT_PCG_NO_FUSED_DOT=1 timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline --pcg-seeds 1 > gpurun_out/pcg_bench_nofuse.jsonl 2> gpurun_out/pcg_bench_nofuse.err
tail -3 gpurun_out/pcg_tests.log
