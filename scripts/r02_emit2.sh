#!/bin/bash
O=gpurun_out/r02e; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_scan.py tests/test_gpu_multi.py tests/test_gpu_literal.py tests/test_gpu_host_stream.py -q --timeout 300 -x > $O/pytest_scan.log 2>&1; echo "pytest rc=$?" >> $O/pytest_scan.log
tail -3 $O/pytest_scan.log
for a in "" "--dbg 64" "--ctas 1 --stages 3" "--ctas 1 --stages 5" "--ctas 2 --stages 2" "--ctas 2 --stages 2 --items 4" "--ctas 2 --stages 4 --items 4" "--variant 3" "--variant 3 --stages 3" "--defer 48" "--defer 64" "--dbg 2"; do
  echo "== $a" >> $O/sweep.log
  timeout 120 python bench.py --config c2 --no-cpu --no-e2e --no-unfused --steps 10 $a 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'): j=json.loads(l); print(j['ms_per_step'], j['roofline']['frac'])
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $O/sweep.log
done
cat $O/sweep.log
python -c "
import sys; sys.path.insert(0,'.')
import workloads, torch
from tests.planspec import build_gpu_plan
p, ids = build_gpu_plan(workloads.c2_spec(), device=0)
print(p.explain(ids['s2']))
" > $O/explain_c2.txt 2>&1; cat $O/explain_c2.txt
