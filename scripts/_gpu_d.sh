mkdir -p gpurun_out/d
timeout 600 python -m pytest tests/test_gpu_merge.py tests/test_gpu_dist.py -q -m gpu > gpurun_out/d/pytest_merge.log 2>&1; tail -2 gpurun_out/d/pytest_merge.log
for P in 2 8; do P=$P timeout 300 python scripts/merge_bench.py >> gpurun_out/d/merge_bench.log 2>&1; done
P=8 timeout 600 ncu --set full --import-source on --clock-control none -k regex:'k_mp_merge' -s 4 -c 1 -o gpurun_out/d/merge -f python scripts/merge_bench.py > gpurun_out/d/ncu_merge.log 2>&1
cat gpurun_out/d/merge_bench.log
