mkdir -p gpurun_out
PM_LS_SPARSE=0 PM_MAX_ROUNDS=1 timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_ls_trap -c 1 -o gpurun_out/trap_full -f python tools/trap_prof.py 4 > gpurun_out/trap_ncu.log 2>&1
echo rc=$?
