mkdir -p gpurun_out; rm -f gpurun_out/ab.log
for v in 1 1g 2 2g 3 3g; do echo "== $v" >> gpurun_out/ab.log; AP_HEUR_POOL=$v timeout 120 python tools/c5_once.py 3 2>&1 | tail -2 >> gpurun_out/ab.log; done
cat gpurun_out/ab.log
