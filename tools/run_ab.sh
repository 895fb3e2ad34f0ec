timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "trap_every_round or trap_chunks or local_search_config" -p no:cacheprovider 2>&1 | tail -1
for rep in 1 2; do for L in tools/libpm_base.so paper_conf_ipps_yangin17_b200/libpm.so; do echo "$L"; PM_LIB=$L REPS=7 timeout 300 python tools/ls_bench.py 3,4 trap 2>&1 | cut -c1-60; done; done
