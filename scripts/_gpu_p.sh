mkdir -p gpurun_out/p
OUT=gpurun_out/p STEPS=20 SPECS="--config c2|--config c1" KNOBS="|--variant 11|--variant 9 --stages 2" bash scripts/knob_sweep.sh > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_scan.py -q -m gpu -x -k "c2" > gpurun_out/p/pytest.log 2>&1; tail -n 2 gpurun_out/p/pytest.log
cat gpurun_out/p/sweep.log
