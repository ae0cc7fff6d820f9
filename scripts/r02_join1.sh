#!/bin/bash
O=gpurun_out/r02s; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_agg_join.py tests/test_gpu_literal.py -q --timeout 300 -x > $O/pytest_join.log 2>&1; echo "pytest rc=$?" >> $O/pytest_join.log
tail -30 $O/pytest_join.log
for c in c3 c5 cc; do
  timeout 300 python bench.py --config $c --no-cpu --no-e2e --steps 10 > $O/bench_$c.log 2>&1
  python -c "import json,sys
for l in open('$O/bench_$c.log'):
  if l.startswith('{'): j=json.loads(l); print('$c', j['ms_per_step'], j['roofline']['frac'], j.get('unfused',{}).get('ms_per_step'))" 
  tail -3 $O/bench_$c.log | grep -i error
done
