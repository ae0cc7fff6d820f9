#!/bin/bash
# C3 diagnostics: expansion phase stamps, ablations (dbg 2 = expansion streams tiles only, dbg 1 = no look-back)
mkdir -p gpurun_out
timeout 300 python scripts/phases.py 0 0 0 0 c3 > gpurun_out/phases_c3.log 2>&1
for v in "" "--dbg 2" "--dbg 1"; do
  echo "== $v" >> gpurun_out/c3var.log
  timeout 300 python bench.py --config c3 --no-e2e --no-cpu --no-unfused $v | python -c "import json,sys; j=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(j['ms_per_step'], j['roofline']['frac'])" >> gpurun_out/c3var.log 2>&1
done
cat gpurun_out/c3var.log; tail -3 gpurun_out/phases_c3.log
