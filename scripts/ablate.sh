#!/bin/bash
# ablations of the C2 scan kernel: full / no look-back / stream only, several stage counts
mkdir -p gpurun_out
for dbg in 0 1 2; do for sc in "0 0 0" "2 1 1" "4 1 2" "6 1 2" "2 2 1" "3 2 1" "2 3 1"; do
  set -- $sc
  echo -n "dbg=$dbg stages=$1 ctas=$2 defer=$3 " >> gpurun_out/ablate.log
  timeout 120 python bench.py --steps 10 --warmup 3 --no-e2e --no-unfused --no-cpu --stages $1 --ctas $2 --defer $3 --dbg $dbg 2>&1 | python -c "import sys,json; l=[x for x in sys.stdin if x.startswith('{')]; j=json.loads(l[-1]) if l else {}; print(j.get('ms_per_step'), j.get('roofline',{}).get('frac'))" >> gpurun_out/ablate.log
done; done
