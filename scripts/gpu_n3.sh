#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_setops.py -m gpu -q -x > gpurun_out/pt_set.log 2>&1; tail -3 gpurun_out/pt_set.log
for op in union intersect difference; do
  timeout 300 python bench.py --config cs --setop $op --no-unfused --no-e2e > gpurun_out/bench_cs_$op.log 2>&1
  python -c "import json; j=json.loads(open('gpurun_out/bench_cs_$op.log').read().strip().splitlines()[-1]); print('$op', j['ms_per_step'], j['roofline']['frac'], j['config']['output_rows_per_gpu'], j.get('cpu_baseline',{}).get('value'))" || tail -5 gpurun_out/bench_cs_$op.log
done
