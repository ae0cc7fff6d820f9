#!/bin/bash
mkdir -p gpurun_out
for sc in "0 0 0" "1 2 3" "1 2 2" "1 1 5" "1 1 6"; do
  set -- $sc
  echo -n "gring=$1 ctas=$2 stages=$3 " >> gpurun_out/sweep.log
  timeout 120 python bench.py --steps 10 --warmup 3 --no-e2e --no-unfused --no-cpu --gring $1 --ctas $2 --stages $3 2>&1 | python -c "import sys,json; l=[x for x in sys.stdin if x.startswith('{')]; j=json.loads(l[-1]) if l else {}; print(j.get('ms_per_step'), j.get('roofline',{}).get('frac'))" >> gpurun_out/sweep.log
done
