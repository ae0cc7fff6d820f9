#!/bin/bash
# round-end evidence: smoke, every GPU test, one bench line per config, launch lists
# and ncu --set full captures of the dominant kernels.  Reports stay in /tmp on the
# box (too big to ship back); their summaries go to gpurun_out/profiles_out/.
mkdir -p gpurun_out/profiles_out
CONFIGS="${CONFIGS:-c2 c1 c3 c4 cd cs c5}" bash scripts/gpu_all.sh > gpurun_out/all.log 2>&1
for spec in ${PROFS:-"c4:k_scan_chain:1:1:22800000360" "cd:k_scan_chain:1:1:0" "cs:k_set_op:1:1:0" "c2:k_scan_chain:1:1:10200709052"}; do
  IFS=: read CFG KREGEX SKIP CNT ALG <<< "$spec"
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' -c 60 --csv \
      --log-file gpurun_out/launches_${CFG}.csv \
      python bench.py --config $CFG --steps 3 --warmup 1 --no-e2e --no-cpu --no-unfused --no-sweep > gpurun_out/ncu_launch_${CFG}.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$KREGEX" -s $SKIP -c $CNT \
      -o /tmp/prof_${CFG} -f \
      python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu --no-sweep > gpurun_out/ncu_full_${CFG}.log 2>&1
  RW_PROFILE_DIR=gpurun_out/profiles_out python scripts/summarize_ncu.py /tmp/prof_${CFG}.ncu-rep ${RW_ROUND_TAG:-r01e}_${CFG}_${KREGEX} $CFG $ALG > /dev/null 2>&1
  echo "$CFG prof rc=$?"
done
