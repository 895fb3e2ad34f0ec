for c in 3 4; do echo "cfg$c"; timeout 300 python tools/sp_rounds.py $c trap 2>&1 | tail -12; done > gpurun_out/sp.txt 2>&1
cat gpurun_out/sp.txt
