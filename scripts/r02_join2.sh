#!/bin/bash
O=gpurun_out/r02s; mkdir -p $O
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base function -k regex:'^k_' -c 40 --csv \
    --log-file $O/launches_c3.csv python bench.py --config c3 --steps 2 --warmup 1 --no-e2e --no-cpu --no-unfused > $O/ncu_launch_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:'k_jmatch|k_join_emit' -s 2 -c 2 \
    -o $O/prof_c3 -f python bench.py --config c3 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu > $O/ncu_c3.log 2>&1
