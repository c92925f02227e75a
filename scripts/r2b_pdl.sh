#!/bin/bash
# PDL A/B (ABFT_NO_PDL=1) + full GPU suite
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/full_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/full_tests.log
rm -f gpurun_out/pdl.log
for rep in 1 2; do
for P in 1 0; do
  for w in 7pt128 7pt192 27pt256 5pt64; do
    echo -n "nopdl=$P $w: " >> gpurun_out/pdl.log
    if [ $P = 1 ]; then E="ABFT_NO_PDL=1"; else E="ABFT_X=0"; fi
    env $E timeout 300 python bench.py --no-cpu-baseline --steps 200 --workload $w 2>&1 | python -c "import sys,json; L=[l for l in sys.stdin if l.startswith('{')]; d=json.loads(L[-1]) if L else None; print(d and (d['value'], d['ms_per_step'], d['plain_ms'], d['roofline']['launch_ms'], d['ft_overhead_pct']))" >> gpurun_out/pdl.log 2>&1
  done
done
done
ABFT_NO_PDL=1 timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline --pcg-seeds 1 > gpurun_out/pcg_nopdl.jsonl 2> gpurun_out/pcg_nopdl.err
timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline --pcg-seeds 1 > gpurun_out/pcg_pdl.jsonl 2> gpurun_out/pcg_pdl.err
tail -3 gpurun_out/full_tests.log; cat gpurun_out/pdl.log
for f in gpurun_out/pcg_nopdl.jsonl gpurun_out/pcg_pdl.jsonl; do python -c "
import json,sys
d=json.loads([l for l in open(sys.argv[1]) if l.startswith('{')][-1])
print(sys.argv[1], {k:(v['ms'],v['iters']) for k,v in d['results'].items() if k.endswith('lam0')})" $f; done
