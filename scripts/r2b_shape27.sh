#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
rm -f gpurun_out/shape27.log
run() { tag=$1; shift
  for w in 27pt128 27pt256; do
    echo -n "$tag $w: " >> gpurun_out/shape27.log
    env "$@" timeout 300 python bench.py --no-cpu-baseline --steps 60 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['ft_overhead_pct'], d['roofline']['kernel']))" >> gpurun_out/shape27.log 2>&1
  done
}
run base ABFT_X=0
run g2x4 ABFT_STREAM_G=2 ABFT_STREAM_SMEM_KB=56
run g8x1 ABFT_STREAM_G=8 ABFT_STREAM_SMEM_KB=227
run g2x3 ABFT_STREAM_G=2 ABFT_STREAM_SMEM_KB=74
run g4x2ns3 ABFT_STREAM_G=4 ABFT_STREAM_SMEM_KB=150
cat gpurun_out/shape27.log
