mkdir -p gpurun_out/c
timeout 600 python -m pytest tests/test_gpu_merge.py tests/test_gpu_dist.py -q -m gpu > gpurun_out/c/pytest_merge.log 2>&1; tail -2 gpurun_out/c/pytest_merge.log
for P in 2 8; do P=$P timeout 300 python scripts/merge_bench.py >> gpurun_out/c/merge_bench.log 2>&1; done
P=8 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_mp' -c 12 --csv --log-file gpurun_out/c/launches_merge.csv python scripts/merge_bench.py > /dev/null 2>&1
OUT=gpurun_out/c STEPS=20 SPECS="--config c2|--config c3|--config c5" KNOBS="|--variant 6|--variant 3" bash scripts/knob_sweep.sh > /dev/null 2>&1
cat gpurun_out/c/merge_bench.log gpurun_out/c/sweep.log
