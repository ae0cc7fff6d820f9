#!/bin/bash
# input stages / CTAs per SM / ring KB sweep of the fused chain; $1 = config, $2 = dbg
CFG=${1:-c2}
DBG=${2:-0}
mkdir -p gpurun_out
for sc in "0 0 0" "2 2 0" "2 2 24" "1 2 0" "3 1 0" "2 1 0" "4 1 0" "3 1 64"; do
  set -- $sc
  echo -n "cfg=$CFG dbg=$DBG stages=$1 ctas=$2 ringKB=$3 " >> gpurun_out/sweep.log
  timeout 120 python bench.py --config $CFG --steps 10 --warmup 3 --no-e2e --no-unfused --no-cpu --stages $1 --ctas $2 --defer $3 --dbg $DBG 2>&1 | python -c "import sys,json; l=[x for x in sys.stdin if x.startswith('{')]; j=json.loads(l[-1]) if l else {}; print(j.get('ms_per_step'), j.get('roofline',{}).get('frac'))" >> gpurun_out/sweep.log
done
