#!/bin/bash
O=gpurun_out/r02ah; mkdir -p $O
for c in "--config c4 --gring 3" "--config c2 --gring 3" "--config c2"; do
  echo "== $c" >> $O/sweep.log
  timeout 300 python bench.py $c --no-cpu --no-e2e --no-sweep --steps 10 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'):
    j=json.loads(l); print(round(j['ms_per_step'],4), round(j['roofline']['frac'],3), 'unfused', round(j.get('unfused',{}).get('ms_per_step',0),4))
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $O/sweep.log
done
cat $O/sweep.log
