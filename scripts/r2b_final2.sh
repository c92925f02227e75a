#!/bin/bash
# round-2 final evidence: GPU suite, smoke, bench lines, sweeps, launch list,
# ncu summaries (reports summarised on the box), compute-sanitizer
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/ncu gpurun_out/final
F=gpurun_out/final
timeout 1500 python -m pytest tests -m gpu -q > $F/gpu_tests.log 2>&1; echo "tests rc=$?" >> $F/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $F/smoke.log 2>&1; echo "smoke rc=$?" >> $F/smoke.log
timeout 600 python bench.py > $F/bench_default.log 2>&1
for W in 27pt256 rmat24 27pt128 5pt64 7pt192 rmat20; do timeout 400 python bench.py --no-cpu-baseline --steps 50 --workload $W > $F/bench_$W.log 2>&1; done
timeout 900 python bench.py --lam-sweep --workload 7pt128 --steps 200 --warmup 10 > $F/lam_7pt128.log 2>&1
timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline > $F/pcg.log 2>&1
timeout 600 python bench.py --pcg-dist --steps 1 --warmup 3 --no-cpu-baseline > $F/pcg_dist.log 2>&1
timeout 600 python bench.py --compare --workload 7pt128 --steps 100 --no-cpu-baseline > $F/compare_7pt128.log 2>&1
timeout 600 python bench.py --strong --workload 27pt256 --steps 20 --warmup 3 --no-cpu-baseline > $F/strong_27pt256.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $F/launches_7pt128.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $F/ncu_launch.log 2>&1
python scripts/launch_summary.py $F/launches_7pt128.csv > $F/launches_7pt128_summary.txt 2>&1
KREGEX="k_stream<\(bool\)1, \(bool\)0" W=7pt128 TAG=stream_prot_7pt128 SKIP=3 UNITS=65536 bash scripts/ncu_one.sh
KREGEX="k_stream<\(bool\)0, \(bool\)0" W=7pt128 TAG=stream_plain_7pt128 SKIP=3 UNITS=65536 bash scripts/ncu_one.sh
KREGEX="k_stream<\(bool\)1, \(bool\)0" W=27pt256 TAG=stream_prot_27pt256 SKIP=3 UNITS=524288 bash scripts/ncu_one.sh
KREGEX="k_irr<\(bool\)1" W=rmat24 TAG=irr_rmat24 SKIP=3 UNITS=1 bash scripts/ncu_one.sh

tail -3 $F/gpu_tests.log; tail -2 $F/smoke.log
for f in $F/bench_*.log; do echo "== $f"; grep '^{' $f | tail -1 | cut -c1-300; done

timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv --log-file $F/launches_rmat24.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --workload rmat24 > $F/ncu_launch_rmat.log 2>&1
python scripts/launch_summary.py $F/launches_rmat24.csv > $F/launches_rmat24_summary.txt 2>&1
