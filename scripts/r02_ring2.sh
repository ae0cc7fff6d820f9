#!/bin/bash
O=gpurun_out/r02ac; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_scan.py tests/test_gpu_multi.py tests/test_gpu_host_stream.py tests/test_gpu_literal.py -q --timeout 300 -x > $O/pytest.log 2>&1; grep -E "passed|failed|FAILED" $O/pytest.log | tail -5
for a in "--config c2" "--config c2 --gring 9" "--config c2 --variant 4" "--config c1 --rows 1073741824" "--config cd"; do
  echo "== $a" >> $O/sweep.log
  timeout 300 python bench.py $a --no-cpu --no-e2e --steps 10 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'):
    j=json.loads(l); print(j['ms_per_step'], round(j['roofline']['frac'],3), 'unfused', j.get('unfused',{}).get('ms_per_step'))
    if 'sweeps' in j: print({k: round(v['fused_ms'],3) for k,v in j['sweeps']['selectivity'].items()}, {k: round(v['unfused_ms'],3) for k,v in j['sweeps']['selectivity'].items()})
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $O/sweep.log
done
cat $O/sweep.log
