timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sparse or local_search" 2>&1 | tail -2
for T in 256 1024; do echo "T=$T"; PM_LS_SPARSE_T=$T REPS=5 timeout 300 python tools/ls_bench.py 1,2 window 2>&1 | tail -2; done
for T in 1024 4096; do echo "T=$T"; PM_LS_SPARSE_T=$T REPS=2 timeout 300 python tools/ls_bench.py 3 class 2>&1 | tail -1; done
PM_LS_SPARSE_T=1024 timeout 120 python tools/sp_rounds.py 2 window
PM_LS_SPARSE_T=4096 timeout 300 python tools/sp_rounds.py 3 class
