mkdir -p gpurun_out/e
timeout 600 python -m pytest tests/test_gpu_merge.py tests/test_gpu_dist.py -q -m gpu > gpurun_out/e/pytest_merge.log 2>&1; tail -2 gpurun_out/e/pytest_merge.log
for P in 2 8; do P=$P timeout 300 python scripts/merge_bench.py >> gpurun_out/e/merge_bench.log 2>&1; done
OUT=gpurun_out/e STEPS=20 SPECS="--config c2" KNOBS="|--variant 4 --ctas 2|--variant 2 --ctas 2|--variant 4 --ctas 1" bash scripts/knob_sweep.sh > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_scan.py tests/test_gpu_fullsize.py -q -m gpu -x > gpurun_out/e/pytest_scan.log 2>&1; tail -2 gpurun_out/e/pytest_scan.log
cat gpurun_out/e/merge_bench.log gpurun_out/e/sweep.log
