#!/bin/bash
timeout 600 python -m pytest tests/test_gpu_scan.py -m gpu -q -x > gpurun_out/pt.log 2>&1; tail -n 1 gpurun_out/pt.log
for a in "" "--variant 8 --items 16 --ctas 4" "--variant 8 --items 16 --ctas 3" "--variant 8 --items 16 --ctas 2"; do
  for c in c2 cd; do
  timeout 300 python bench.py --config $c $a --no-cpu --no-e2e --no-unfused --steps 10 > gpurun_out/b.log 2>&1
  python -c "import json; j=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$c [$a]', round(j['ms_per_step'],3), round(j['roofline']['frac'],3))" || tail -n 3 gpurun_out/b.log
  done
done
