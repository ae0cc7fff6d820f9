mkdir -p gpurun_out/s
timeout 900 python -m pytest tests/test_gpu_merge.py tests/test_gpu_dist.py -q -m gpu -x > gpurun_out/s/pytest.log 2>&1; tail -n 3 gpurun_out/s/pytest.log
OUT=gpurun_out/s STEPS=20 SPECS="--config c5|--config c3" KNOBS="|--stages 1" bash scripts/knob_sweep.sh > /dev/null 2>&1
cat gpurun_out/s/sweep.log
