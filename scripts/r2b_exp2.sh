#!/bin/bash
# k_hub occupancy variants on R-MAT; refresh PCG / sharded / strong lines
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
P=paper_conf_dsn_schollbkw16_b200
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "popularity or irregular or hub or rmat or bench_workloads" > gpurun_out/exp2_tests.log 2>&1; echo "rc=$?" >> gpurun_out/exp2_tests.log
rm -f gpurun_out/exp2.log
for lib in libabft.so libabft_h4.so libabft_h6u8.so; do
  for w in rmat24 rmat22; do
    echo -n "$lib $w: " >> gpurun_out/exp2.log
    ABFT_LIB=$PWD/$P/$lib timeout 300 python bench.py --no-cpu-baseline --steps 30 --workload $w > gpurun_out/exp2_${lib}_$w.log 2>&1
    python -c "import sys,json; L=[l for l in open(sys.argv[1]) if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct'], d['gpu_launches']))" gpurun_out/exp2_${lib}_$w.log >> gpurun_out/exp2.log 2>&1
  done
done
timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/pcg.jsonl 2> gpurun_out/pcg.err
timeout 600 python bench.py --pcg-dist --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/pcg_dist.log 2>&1
timeout 600 python bench.py --strong --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/strong.log 2>&1
tail -2 gpurun_out/exp2_tests.log; cat gpurun_out/exp2.log
tail -c 600 gpurun_out/pcg.jsonl; tail -c 600 gpurun_out/pcg_dist.log; tail -c 800 gpurun_out/strong.log
