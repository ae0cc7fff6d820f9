#!/bin/bash
CFG=${1:-c2}
mkdir -p gpurun_out
for sc in "0 0 0" "1 3 0" "1 3 40" "2 2 0" "3 1 0"; do
  set -- $sc
  echo -n "cfg=$CFG stages=$1 ctas=$2 ringKB=$3 " >> gpurun_out/sweep.log
  timeout 120 python bench.py --config $CFG --steps 10 --warmup 3 --no-e2e --no-unfused --no-cpu --stages $1 --ctas $2 --defer $3 2>&1 | python -c "import sys,json; l=[x for x in sys.stdin if x.startswith('{')]; j=json.loads(l[-1]) if l else {}; print(j.get('ms_per_step'), j.get('roofline',{}).get('frac'))" >> gpurun_out/sweep.log
done
