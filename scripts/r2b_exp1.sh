#!/bin/bash
# k_stream SHORT variants (3 CTAs/SM; depth-3 gather pipeline) + R-MAT 24 ncu with popularity order
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/ncu
P=paper_conf_dsn_schollbkw16_b200
ABFT_LIB=$PWD/$P/libabft_d3.so timeout 900 python -m pytest tests/test_gpu_stream.py -x -q > gpurun_out/d3_tests.log 2>&1; echo "rc=$?" >> gpurun_out/d3_tests.log
run() { # tag env... 
  tag=$1; shift
  for w in 7pt128 7pt192; do
    echo -n "$tag $w: " >> gpurun_out/exp1.log
    env "$@" timeout 300 python bench.py --no-cpu-baseline --steps 300 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct'], d['roofline']['kernel']))" >> gpurun_out/exp1.log 2>&1
  done
}
rm -f gpurun_out/exp1.log
run base ABFT_LIB=$PWD/$P/libabft.so
run d3 ABFT_LIB=$PWD/$P/libabft_d3.so
run m3 ABFT_LIB=$PWD/$P/libabft_m3.so ABFT_STREAM_SMEM_KB=74
run m3g4 ABFT_LIB=$PWD/$P/libabft_m3.so ABFT_STREAM_SMEM_KB=74 ABFT_STREAM_G=4
run base2 ABFT_LIB=$PWD/$P/libabft.so
KREGEX="k_hub" W=rmat24 TAG=hub24 SKIP=3 UNITS=1 bash scripts/ncu_one.sh
KREGEX="k_irr<\(bool\)1" W=rmat24 TAG=irr24 SKIP=3 UNITS=1 bash scripts/ncu_one.sh
KREGEX="k_xperm" W=rmat24 TAG=xperm24 SKIP=3 UNITS=1 bash scripts/ncu_one.sh
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_rmat24.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --workload rmat24 > gpurun_out/ncu_launch_rmat.log 2>&1
python scripts/launch_summary.py gpurun_out/launches_rmat24.csv > gpurun_out/launches_rmat24_summary.txt
tail -2 gpurun_out/d3_tests.log; cat gpurun_out/exp1.log; head -12 gpurun_out/launches_rmat24_summary.txt
