#!/bin/bash
timeout 900 python -m pytest tests/test_gpu_agg_join.py tests/test_gpu_dist.py -m gpu -q -x > gpurun_out/pt.log 2>&1; tail -n 1 gpurun_out/pt.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "c3" > gpurun_out/pt2.log 2>&1; tail -n 1 gpurun_out/pt2.log
for c in c3 c5; do for a in "" "--dbg 4096"; do
  timeout 300 python bench.py --config $c $a --no-cpu --no-e2e --no-unfused --steps 10 > gpurun_out/b.log 2>&1
  python -c "import json; j=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$c [$a]', round(j['ms_per_step'],3), round(j['roofline']['frac'],3), j['gpu_launches'])" || tail -n 3 gpurun_out/b.log
done; done
