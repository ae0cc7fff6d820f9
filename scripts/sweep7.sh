#!/bin/bash
mkdir -p gpurun_out
for sc in "0 0 0 0" "0 2 3 8" "0 2 4 6" "0 2 3 6" "0 2 4 5" "2 0 0 0"; do
  set -- $sc
  echo -n "gring=$1 ctas=$2 stages=$3 items=$4 " >> gpurun_out/sweep.log
  timeout 120 python bench.py --steps 10 --warmup 3 --no-e2e --no-unfused --no-cpu --gring $1 --ctas $2 --stages $3 --items $4 2>&1 | python -c "import sys,json; l=[x for x in sys.stdin if x.startswith('{')]; j=json.loads(l[-1]) if l else {}; print(j.get('ms_per_step'), j.get('roofline',{}).get('frac'))" >> gpurun_out/sweep.log
done
