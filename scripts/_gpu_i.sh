mkdir -p gpurun_out/i
timeout 1200 python -m pytest tests/test_gpu_agg_join.py tests/test_gpu_join2.py tests/test_gpu_dist.py tests/test_gpu_legality.py -q -m gpu -x > gpurun_out/i/pytest_join.log 2>&1; tail -n 3 gpurun_out/i/pytest_join.log
OUT=gpurun_out/i STEPS=20 SPECS="--config c3|--config c5|--config cc" KNOBS="" bash scripts/knob_sweep.sh > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -m gpu -x -k "c3 or c5 or join" > gpurun_out/i/pytest_full.log 2>&1; tail -n 3 gpurun_out/i/pytest_full.log
cat gpurun_out/i/sweep.log
