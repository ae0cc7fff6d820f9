#!/bin/bash
# r02 baseline: source-level ncu captures of the C2 scan and the C3 join kernels
mkdir -p gpurun_out/r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r02a/gpu.txt 2>&1
timeout 300 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/r02a/bench_c2.log 2>&1
timeout 300 python bench.py --config c3 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/r02a/bench_c3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:k_scan_chain -s 2 -c 1 \
    -o gpurun_out/r02a/prof_c2 -f python bench.py --config c2 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu > gpurun_out/r02a/ncu_c2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:'k_scan_chain|k_join_runs' -s 4 -c 3 \
    -o gpurun_out/r02a/prof_c3 -f python bench.py --config c3 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu > gpurun_out/r02a/ncu_c3.log 2>&1
ls -la gpurun_out/r02a
