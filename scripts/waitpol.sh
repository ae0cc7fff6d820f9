#!/bin/bash
for a in "" "--variant 7 --items 6" "" "--variant 7 --items 6"; do
  for c in c2 cd; do
  timeout 300 python bench.py --config $c $a --no-cpu --no-e2e --no-unfused --steps 10 > gpurun_out/b.log 2>&1
  python -c "import json; j=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$c [$a]', round(j['ms_per_step'],3), round(j['roofline']['frac'],3))" || tail -n 2 gpurun_out/b.log
  done
done
