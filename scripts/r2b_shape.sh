#!/bin/bash
# k_stream chunk / ring shapes at equal consumer warps and bytes in flight per SM
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
rm -f gpurun_out/shape.log
run() { tag=$1; shift
  for w in 7pt128 7pt192; do
    echo -n "$tag $w: " >> gpurun_out/shape.log
    env "$@" timeout 300 python bench.py --no-cpu-baseline --steps 200 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct'], d['roofline']['kernel']))" >> gpurun_out/shape.log 2>&1
  done
}
for rep in 1 2; do
run base ABFT_X=0
run g4x4cta ABFT_STREAM_G=4 ABFT_STREAM_SMEM_KB=56
run g2x8cta ABFT_STREAM_G=2 ABFT_STREAM_SMEM_KB=28
run g4x3cta ABFT_STREAM_G=4 ABFT_STREAM_SMEM_KB=74
done
cat gpurun_out/shape.log
