#!/bin/bash
# r01f knob sweep: CTAs/SM for the join configs, tile rows for the small C1 case
mkdir -p gpurun_out
for spec in "c3 --ctas 1" "c3 --ctas 2" "c5 --ctas 1" "c5 --ctas 2" "c1 --items 4" "c1 --items 8" "cc --ctas 1"; do
  r=$(timeout 300 python bench.py --config $spec --no-e2e --no-cpu --no-unfused 2>&1 | python -c "import json,sys; j=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print(round(j['ms_per_step'],3), round(j['roofline']['frac'],4))" 2>&1)
  echo "$spec: $r" >> gpurun_out/sweep8.log
done
cat gpurun_out/sweep8.log
