#!/bin/bash
# TRAP development probe: parity tests, phase profile, whole-search timings
out=gpurun_out/$1; mkdir -p $out
timeout 900 python -m pytest tests -x -q -m gpu -k "trap or local_search" > $out/pytest.log 2>&1; echo rc=$? >> $out/pytest.log
for v in 0 1 3; do for cm in 0 1; do
  PM_TRAP_CLUSTER=$cm PM_TRAP_V=$v PM_LS_SPARSE=0 timeout 120 python tools/trap_prof.py 1,2,3,4 > $out/prof_v${v}_c$cm.txt 2>&1
done; done
for v in 0 1 3; do PM_TRAP_V=$v REPS=5 timeout 300 python tools/ls_bench.py 1,2,3,4 trap > $out/ls_v$v.txt 2>&1; done
