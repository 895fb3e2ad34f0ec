mkdir -p gpurun_out
for pr in 3 1; do for sp in ${SPECS:-0 1}; do echo "PROF=$pr SPEC=$sp"; PM_TRAP_PROF=$pr PM_TRAP_SPEC=$sp PM_LS_SPARSE=0 timeout 300 python tools/trap_prof.py ${CFGS:-3,4} 2>&1 | tail -2; done; done > gpurun_out/prof.txt 2>&1
cat gpurun_out/prof.txt
