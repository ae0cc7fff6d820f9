#!/bin/bash
# launch list of this repo's kernels + one full ncu capture of the dominant kernel
# usage: scripts/gpu_prof.sh <config> <kernel-regex>
CFG=${1:-c2}
KREGEX=${2:-k_scan_chain}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base function -k regex:'^k_' -c 60 --csv \
    --log-file gpurun_out/launches_${CFG}.csv \
    python bench.py --config $CFG --steps 3 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_${CFG}.log 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:$KREGEX -s 2 -c 1 \
    -o gpurun_out/prof_${CFG} -f \
    python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu > gpurun_out/ncu_full_${CFG}.log 2>&1
echo done
