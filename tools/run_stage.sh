mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "trap or sparse or walk or local_search" -p no:cacheprovider > gpurun_out/st_tests.txt 2>&1; echo "rc=$?" >> gpurun_out/st_tests.txt
tail -2 gpurun_out/st_tests.txt
REPS=5 timeout 300 python tools/ls_bench.py 1,2,3,4 trap 2>&1
