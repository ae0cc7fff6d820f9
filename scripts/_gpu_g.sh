mkdir -p gpurun_out/g
timeout 900 python -m pytest tests/test_gpu_agg_join.py -q -m gpu -x -k "q1" > gpurun_out/g/pytest_q1.log 2>&1; tail -n 3 gpurun_out/g/pytest_q1.log
OUT=gpurun_out/g STEPS=20 SPECS="--config c4" KNOBS="|--agg-mode 2" bash scripts/knob_sweep.sh > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum --clock-control none -k regex:'k_scan_chain' -c 2 --csv --log-file gpurun_out/g/c4_metrics.csv python bench.py --config c4 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu --no-sweep > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -m gpu -x -k "q1 or c4 or agg" > gpurun_out/g/pytest_full.log 2>&1; tail -n 3 gpurun_out/g/pytest_full.log
cat gpurun_out/g/sweep.log
