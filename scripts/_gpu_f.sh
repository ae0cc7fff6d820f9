mkdir -p gpurun_out/f
timeout 900 python -m pytest tests/test_gpu_scan.py -q -m gpu -x -k "team or c2" > gpurun_out/f/pytest_team.log 2>&1; tail -n 3 gpurun_out/f/pytest_team.log
OUT=gpurun_out/f STEPS=20 SPECS="--config c2" KNOBS="|--variant 7|--variant 8|--variant 7 --stages 4|--variant 7 --stages 6|--variant 8 --stages 4" bash scripts/knob_sweep.sh > /dev/null 2>&1
cat gpurun_out/f/sweep.log
