#!/bin/bash
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -k "pcg or cg1" > gpurun_out/fold_tests.log 2>&1; echo "rc=$?" >> gpurun_out/fold_tests.log
rm -f gpurun_out/fold.log
for rep in 1 2; do
  ABFT_PCG_NO_FIN_DOT=1 timeout 300 python scripts/pcg_time.py | sed 's/^/nofold /' >> gpurun_out/fold.log 2>&1
  timeout 300 python scripts/pcg_time.py | sed 's/^/fold /' >> gpurun_out/fold.log 2>&1
done
timeout 900 python bench.py --pcg --steps 1 --warmup 3 --no-cpu-baseline --pcg-seeds 1 > gpurun_out/fold_pcg.jsonl 2>/dev/null
tail -2 gpurun_out/fold_tests.log; cat gpurun_out/fold.log
python -c "
import json
d=json.loads([l for l in open('gpurun_out/fold_pcg.jsonl') if l.startswith('{')][-1])
print({k:(v['ms'],v['iters'],v['success_rate']) for k,v in d['results'].items()})"
