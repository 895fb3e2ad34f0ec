mkdir -p gpurun_out
for sp in 1 2; do echo "SPEC=$sp"; PM_TRAP_PROF=3 PM_TRAP_SPEC=$sp PM_LS_SPARSE=0 PM_MAX_ROUNDS=7 timeout 300 python tools/trap_prof.py 2,3,4 2>&1 | tail -3; done > gpurun_out/spec.txt 2>&1
cat gpurun_out/spec.txt
