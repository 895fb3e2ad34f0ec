for T in 128 256 512 1024 2048; do echo "T=$T"; PM_LS_SPARSE_T=$T REPS=3 timeout 300 python tools/ls_bench.py 2,3,4 trap 2>&1 | cut -c1-60; done
for T in 16 32 64 128 256; do echo "T=$T cfg5"; PM_LS_SPARSE_T=$T timeout 300 python tools/ep_bench.py 5 2>&1 | tail -1 | cut -c1-90; done
