# E kernel plan sweep (bn x split-K) at configs 1-3: development probe
mkdir -p gpurun_out
for p in 0 128001 128002 128003 128004 128006 64001 64002 64003 64004 64006 64012; do echo "plan=$p"; PM_SAD_PLAN=$p python tools/e_bench.py ${CFGS:-1,2,3} 2>&1 | grep fused; done > gpurun_out/sad_sweep.txt 2>&1
cat gpurun_out/sad_sweep.txt
