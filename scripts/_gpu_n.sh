mkdir -p gpurun_out/n
timeout 1200 python -m pytest tests/test_gpu_agg_join.py tests/test_gpu_join2.py tests/test_gpu_scan.py -q -m gpu -x > gpurun_out/n/pytest.log 2>&1; tail -n 3 gpurun_out/n/pytest.log
OUT=gpurun_out/n STEPS=20 SPECS="--config c2|--config c5|--config c3|--config cc" KNOBS="|--variant 9" bash scripts/knob_sweep.sh > /dev/null 2>&1
cat gpurun_out/n/sweep.log
