#!/bin/bash
# N1 input-dependence fusion + C4 wide-CTA variants: parity, then bench lines
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python bench.py --config cd --no-cpu > gpurun_out/bench_cd.log 2>&1
timeout 300 python bench.py --config cd --branches 3 --no-cpu --no-e2e > gpurun_out/bench_cd3.log 2>&1
for v in 0 4 5; do
  timeout 300 python bench.py --config c4 --variant $v --no-cpu --no-e2e --no-unfused > gpurun_out/bench_c4_v$v.log 2>&1
done
tail -3 gpurun_out/pytest_gpu.log
