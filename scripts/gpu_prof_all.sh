#!/bin/bash
# launch lists (gpu__time_duration per launch) + one ncu --set full capture of the
# dominant kernels for each config; reports under gpurun_out/
mkdir -p gpurun_out
for spec in ${PROFS:-"c2:k_scan_chain:1:1" "c4:k_scan_chain:1:1" "c3:k_scan_chain|k_join_runs:3:3"}; do
  IFS=: read CFG KREGEX SKIP CNT <<< "$spec"
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' -c 60 --csv \
      --log-file gpurun_out/launches_${CFG}.csv \
      python bench.py --config $CFG --steps 3 --warmup 1 --no-e2e --no-cpu ${BENCH_ARGS} > gpurun_out/ncu_launch_${CFG}.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$KREGEX" -s $SKIP -c $CNT \
      -o gpurun_out/prof_${CFG} -f \
      python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu ${BENCH_ARGS} > gpurun_out/ncu_full_${CFG}.log 2>&1
  echo "$CFG done rc=$?"
done
