#!/bin/bash
mkdir -p gpurun_out
for sc in "0 0 0 0" "3 8 1 2" "3 8 1 0" "2 4 2 2" "2 4 1 4"; do
  set -- $sc
  echo -n "variant=$1 items=$2 ctas=$3 stages=$4 " >> gpurun_out/sweep.log
  timeout 120 python bench.py --steps 10 --warmup 3 --no-e2e --no-unfused --no-cpu --variant $1 --items $2 --ctas $3 --stages $4 2>&1 | python -c "import sys,json; l=[x for x in sys.stdin if x.startswith('{')]; j=json.loads(l[-1]) if l else {}; print(j.get('ms_per_step'), j.get('roofline',{}).get('frac'))" >> gpurun_out/sweep.log
done
