#!/bin/bash
O=gpurun_out/r02h; mkdir -p $O
for a in "" "--variant 3" "--variant 5" "--variant 4" "--variant 3 --dbg 2" "--variant 5 --dbg 2" "--variant 3 --defer 64" "--variant 3 --defer 80"; do
  echo "== $a" >> $O/sweep.log
  timeout 120 python bench.py --config c2 --no-cpu --no-e2e --no-unfused --steps 10 $a 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'): j=json.loads(l); print(j['ms_per_step'], j['roofline']['frac'])
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $O/sweep.log
done
cat $O/sweep.log
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:k_scan_emit -s 2 -c 1 \
    -o $O/prof_v5 -f python bench.py --config c2 --variant 5 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu > $O/ncu_v5.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:k_scan_emit -s 2 -c 1 \
    -o $O/prof_v3 -f python bench.py --config c2 --variant 3 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu > $O/ncu_v3.log 2>&1
