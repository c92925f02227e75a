#!/bin/bash
# final state: GPU suite, smoke, bench lines, PCG, launch lists
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/final3
F=gpurun_out/final3
timeout 1500 python -m pytest tests -m gpu -q > $F/gpu_tests.log 2>&1; echo "tests rc=$?" >> $F/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $F/smoke.log 2>&1; echo "smoke rc=$?" >> $F/smoke.log
timeout 600 python bench.py > $F/bench_default.log 2>&1
for W in 27pt256 rmat24 7pt192 rmat20 27pt128 5pt64; do timeout 400 python bench.py --no-cpu-baseline --steps 50 --workload $W > $F/bench_$W.log 2>&1; done
timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline > $F/pcg.log 2>&1
timeout 600 python bench.py --pcg-dist --steps 1 --warmup 3 --no-cpu-baseline > $F/pcg_dist.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $F/reference.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv --log-file $F/launches_rmat24.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --workload rmat24 > $F/ncu_launch_rmat.log 2>&1
python scripts/launch_summary.py $F/launches_rmat24.csv > $F/launches_rmat24_summary.txt 2>&1
ABFT_PCG_HOST_LOOP=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 20 -c 120 --csv --log-file $F/launches_pcg.csv python scripts/pcg_profile.py 192 1 > $F/ncu_pcg.log 2>&1
python scripts/launch_summary.py $F/launches_pcg.csv > $F/launches_pcg_summary.txt 2>&1
tail -3 $F/gpu_tests.log; tail -2 $F/smoke.log
for f in $F/bench_*.log; do echo "== $f"; grep '^{' $f | tail -1 | cut -c1-200; done
