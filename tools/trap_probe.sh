#!/bin/bash
# TRAP development probe: parity tests, phase profile, timing per variant
out=gpurun_out/$1; mkdir -p $out
timeout 600 python -m pytest tests -x -q -m gpu -k "trap" > $out/pytest.log 2>&1; echo rc=$? >> $out/pytest.log
for v in 0 1 2 3 4; do for g in 1 2 4; do
  PM_TRAP_V=$v PM_TRAP_GSZ=$g PM_LS_SPARSE=0 timeout 120 python tools/trap_prof.py 1,2,3,4 > $out/prof_v${v}_g$g.txt 2>&1
done; done
