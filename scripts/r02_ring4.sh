#!/bin/bash
O=gpurun_out/r02ai2; mkdir -p $O
for c in "--config c2" "--config c1" "--config c1 --rows 1073741824" "--config cd" "--config c3"; do for a in "" "--gring 9" "--gring 8"; do
  echo "== $c $a" >> $O/sweep.log
  timeout 300 python bench.py $c $a --no-cpu --no-e2e --no-sweep --steps 10 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'):
    j=json.loads(l); print(round(j['ms_per_step'],4), round(j['roofline']['frac'],3), 'unfused', round(j.get('unfused',{}).get('ms_per_step',0),4))
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $O/sweep.log
done; done
cat $O/sweep.log
