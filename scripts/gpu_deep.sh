#!/bin/bash
# one gpurun call: new-kernel tests, merge microbench, and ncu --set full captures of
# single launches whose reports are brought back (gpurun_out/deep/*.ncu-rep) for
# source-level reading here (scripts/ncu_src.py)
O=gpurun_out/deep; mkdir -p $O
timeout 900 python -m pytest ${TESTS:-tests/test_gpu_merge.py tests/test_gpu_dist.py} -q -m gpu > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
for P in 2 8; do P=$P timeout 300 python scripts/merge_bench.py >> $O/merge_bench.log 2>&1; done
P=8 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_mp' --csv \
    --log-file $O/launches_merge.csv python scripts/merge_bench.py > $O/ncu_merge.log 2>&1
for spec in ${CAPS:-"c3:k_join_emit:1:1" "c4:k_scan_chain:1:1" "c2:k_scan_emit:1:1" "c3:k_jmatch:1:1"}; do
  IFS=: read CFG KREGEX SKIP CNT <<< "$spec"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$KREGEX" -s $SKIP -c $CNT \
      -o $O/${CFG}_${KREGEX} -f \
      python bench.py --config $CFG --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu --no-sweep ${BENCH_ARGS} > $O/ncu_${CFG}_${KREGEX}.log 2>&1
  echo "$CFG $KREGEX rc=$?" >> $O/caps.log
done
ls -la $O
