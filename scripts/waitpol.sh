#!/bin/bash
timeout 900 python -m pytest tests/test_gpu_scan.py tests/test_gpu_multi.py tests/test_gpu_host_stream.py -m gpu -q -x > gpurun_out/pt.log 2>&1; tail -n 1 gpurun_out/pt.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "c2 or pattern_d" > gpurun_out/pt2.log 2>&1; tail -n 1 gpurun_out/pt2.log
for a in 1 2; do for c in c2 cd c1; do
  timeout 300 python bench.py --config $c --no-cpu --no-e2e --steps 10 > gpurun_out/b.log 2>&1
  python -c "import json; j=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$c', round(j['ms_per_step'],4), round(j['roofline']['frac'],3), j.get('unfused',{}).get('speedup_fused_vs_unfused'))" || tail -n 3 gpurun_out/b.log
done; done
