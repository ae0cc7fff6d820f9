#!/bin/bash
# Knob sweep over bench configurations (one gpurun call).  Each SPEC is a quoted list of
# bench.py arguments; every combination of SPECS x KNOBS is run once and one line
# "ms_per_step frac unfused_ms" is appended to $OUT/sweep.log.  Diagnostic only: these
# lines are not bench values (no clocks check, few steps).
#   OUT=gpurun_out/r02x SPECS="--config c2|--config c3" KNOBS="|--gring 9" bash scripts/knob_sweep.sh
OUT=${OUT:-gpurun_out/sweep}; mkdir -p $OUT
IFS='|' read -ra SPECL <<< "${SPECS:---config c2}"
IFS='|' read -ra KNOBL <<< "${KNOBS:-}"
[ ${#KNOBL[@]} -eq 0 ] && KNOBL=("")
for c in "${SPECL[@]}"; do for a in "${KNOBL[@]}"; do
  echo "== $c $a" >> $OUT/sweep.log
  timeout ${TMO:-300} python bench.py $c $a --no-cpu --no-e2e --no-sweep --steps ${STEPS:-10} ${EXTRA} 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'):
    j=json.loads(l); print(round(j['ms_per_step'],4), round(j['roofline']['frac'],3), 'unfused', round((j.get('unfused') or {}).get('ms_per_step',0),4))
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $OUT/sweep.log
done; done
cat $OUT/sweep.log
