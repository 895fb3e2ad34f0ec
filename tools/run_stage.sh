mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "trap or sparse or walk or local_search" -p no:cacheprovider > gpurun_out/st_tests.txt 2>&1; echo "rc=$?" >> gpurun_out/st_tests.txt
tail -2 gpurun_out/st_tests.txt
REPS=3 timeout 300 python tools/ls_bench.py 2,3,4 trap 2>&1
for pr in 3; do for sp in 1; do PM_TRAP_PROF=$pr PM_TRAP_SPEC=$sp PM_LS_SPARSE=0 timeout 300 python tools/trap_prof.py 3,4 2>&1 | tail -2; done; done
