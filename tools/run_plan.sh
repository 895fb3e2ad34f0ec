for p in 0 128001 64001; do echo "plan=$p"; PM_SAD_PLAN=$p timeout 300 python tools/e_bench.py 3,4 2>&1 | grep cfg; done
