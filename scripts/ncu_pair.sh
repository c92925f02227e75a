#!/bin/bash
# ncu --set full captures of k_lean<CHECK> and k_lean<plain> on the bench workload
cd $GRAFT_REPO_ROOT; O=gpurun_out/${NCU_TAG:-pair}; mkdir -p $O
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:k_lean<.bool.1, .bool.0, .int.1, .int.3>' -s 6 -c 1 -o $O/lean_check -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $O/ncu_check.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:k_lean<.bool.0, .bool.0, .int.1, .int.3>' -s 2 -c 1 -o $O/lean_plain -f python bench.py --steps 3 --warmup 3 --no-cpu-baseline > $O/ncu_plain.log 2>&1
ls -la $O; tail -n 3 $O/ncu_check.log; tail -n 3 $O/ncu_plain.log
