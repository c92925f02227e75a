#!/bin/bash
# round-2 (session b) baseline: full GPU suite, smoke, bench lines, launch list, ncu of k_stream
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/ncu
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/full_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/full_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 400 python bench.py > gpurun_out/bench_default.log 2>&1
for W in 27pt256 rmat24 27pt128 5pt64; do timeout 400 python bench.py --no-cpu-baseline --steps 50 --workload $W > gpurun_out/bench_$W.log 2>&1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
KREGEX="k_stream<\(bool\)1, \(bool\)0" W=7pt128 TAG=stream_prot SKIP=3 bash scripts/ncu_one.sh
KREGEX="k_stream<\(bool\)0, \(bool\)0" W=7pt128 TAG=stream_plain SKIP=3 bash scripts/ncu_one.sh
tail -3 gpurun_out/full_tests.log; tail -2 gpurun_out/smoke.log
for f in gpurun_out/bench_*.log; do echo "== $f"; grep '^{' $f | tail -1 | cut -c1-600; done
