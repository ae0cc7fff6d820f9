#!/bin/bash
# one gpurun call: smoke, gpu tests, bench lines for every config; logs under gpurun_out/
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt 2>&1
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for c in ${CONFIGS:-c2 c1 c3 c4 c5}; do
  timeout 600 python bench.py --config $c ${BENCH_ARGS} > gpurun_out/bench_$c.log 2>&1; echo "bench $c rc=$?" >> gpurun_out/bench_$c.log
done
for f in gpurun_out/smoke.log gpurun_out/pytest_gpu.log gpurun_out/bench_*.log; do tail -n 3 $f; done
