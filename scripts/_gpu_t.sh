mkdir -p gpurun_out/t
timeout 600 python -m pytest tests/test_gpu_scan.py -q -m gpu -x > gpurun_out/t/pytest.log 2>&1; tail -n 2 gpurun_out/t/pytest.log
OUT=gpurun_out/t STEPS=20 SPECS="--config c2|--config c1" KNOBS="" bash scripts/knob_sweep.sh > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'k_scan_emit' -c 2 --csv --log-file gpurun_out/t/c2_dram.csv python bench.py --config c2 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu --no-sweep > /dev/null 2>&1
cat gpurun_out/t/sweep.log; grep -E "dram|duration" gpurun_out/t/c2_dram.csv | cut -d, -f12-16
