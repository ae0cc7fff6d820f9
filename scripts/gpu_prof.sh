#!/bin/bash
# launch list + full ncu capture of the dominant kernel for a config ($1, default c2)
CFG=${1:-c2}
KREGEX=${2:-k_scan_chain}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_${CFG}.csv \
    python bench.py --config $CFG --steps 3 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_${CFG}.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:$KREGEX -s 2 -c 1 -o gpurun_out/prof_${CFG} -f \
    python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu > gpurun_out/ncu_full_${CFG}.log 2>&1
echo done
