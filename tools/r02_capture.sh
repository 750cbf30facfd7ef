#!/bin/bash
# Round-2 evidence on one B200 (run under gpurun from the repo root): GPU tests, ncu
# --set full captures of the dominant sweep, the C5 heuristic pool and the T + master
# evaluation kernel (summarised here: the .ncu-rep files are too large to bring back),
# the bench line (its roofline.ncu block reads the fresh sweep summary), the ncu launch
# list of the bench command, the 2-rank gloo bench on one GPU and a short reference-arm
# run.  Outputs in gpurun_out/.
set -x
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 > $O/r02_pytest.log 2>&1; tail -3 $O/r02_pytest.log
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k "regex:k_sweep_exact<.int.8, unsigned int, .bool.0>" -s 2 -c 1 -o $O/sweep_c4_r2 \
  python bench.py --steps 1 --warmup 3 --no-secondary --no-cpu-baseline > $O/ncu_sweep_r2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_heur_pool -s 0 -c 1 \
  -o $O/heurpool_c5_r2 python tools/c5_once.py 1 > $O/ncu_heur_r2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_eval_fast -s 8 -c 1 \
  -o $O/evalfast_master_c4_r2 python tools/eval_time.py 4 20 > $O/ncu_eval_r2.log 2>&1
python tools/ncu_summary.py $O/sweep_c4_r2.ncu-rep 5569524480 12 --json $O/ncu_sweep_c4.json > $O/r02_ncu_sweep.txt 2>&1
python tools/ncu_summary.py $O/heurpool_c5_r2.ncu-rep 1289183 14 > $O/r02_ncu_heur.txt 2>&1
python tools/ncu_summary.py $O/evalfast_master_c4_r2.ncu-rep 1048576 12 > $O/r02_ncu_evalfast.txt 2>&1
for r in sweep_c4_r2 heurpool_c5_r2 evalfast_master_c4_r2; do
  ncu -i $O/$r.ncu-rep --page source --csv --print-source sass > $O/$r.sass.csv 2>/dev/null
  python - "$O/$r.sass.csv" > $O/$r.opcodes.txt <<'PY'
import csv, sys
from collections import Counter
rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]; ix = {k: i for i, k in enumerate(h)}
c = Counter(); tot = 0
for rr in rows[2:]:
    if len(rr) < len(h): continue
    try: n = int(rr[ix["Instructions Executed"]] or 0)
    except Exception: continue
    src = rr[ix["Source"]].strip()
    op = (src.split()[1] if src.startswith("@") else src.split()[0]).split(".")[0]
    c[op] += n; tot += n
print("total warp-instructions", tot)
for op, n in c.most_common(30): print(op, n)
PY
  rm -f $O/$r.sass.csv $O/$r.ncu-rep
done
# the bench reads profiles/ncu_sweep_c4.json for roofline.ncu / traffic: use this capture's
[ -s $O/ncu_sweep_c4.json ] && cp $O/ncu_sweep_c4.json profiles/ncu_sweep_c4.json
timeout 900 python bench.py > $O/r02_bench.json 2> $O/r02_bench.err; tail -c 300 $O/r02_bench.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/r02_bench_under_ncu.log 2>&1
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29533 bench.py --gpus 2 --backend gloo --device-override 0 --steps 5 --warmup 3 \
  --no-cpu-baseline > $O/r02_bench_2rank_gloo.json 2> $O/r02_bench_2rank_gloo.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/r02_bench_reference.json 2>&1
ls -la $O
