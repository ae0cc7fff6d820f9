#!/bin/bash
CFG=${1:-c2}
mkdir -p gpurun_out
for sc in "0 0 0" "8 2 2" "6 2 2" "6 2 3" "5 2 2" "5 2 3" "5 2 4" "4 2 4" "4 2 5"; do
  set -- $sc
  echo -n "cfg=$CFG items=$1 ctas=$2 stages=$3 " >> gpurun_out/sweep.log
  timeout 120 python bench.py --config $CFG --steps 10 --warmup 3 --no-e2e --no-unfused --no-cpu --items $1 --ctas $2 --stages $3 2>&1 | python -c "import sys,json; l=[x for x in sys.stdin if x.startswith('{')]; j=json.loads(l[-1]) if l else {}; print(j.get('ms_per_step'), j.get('roofline',{}).get('frac'))" >> gpurun_out/sweep.log
done
