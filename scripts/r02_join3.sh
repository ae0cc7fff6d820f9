#!/bin/bash
O=gpurun_out/r02u; mkdir -p $O
for a in "" "--variant 7" "--variant 8"; do
  for c in c3 c5; do
  echo "== $c $a" >> $O/sweep.log
  timeout 120 python bench.py --config $c --no-cpu --no-e2e --no-unfused --steps 5 $a 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'): j=json.loads(l); print(j['ms_per_step'], j['roofline']['frac'])
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $O/sweep.log
  done
done
cat $O/sweep.log
