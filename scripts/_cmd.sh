mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_agg_join.py tests/test_gpu_scan.py -m gpu -q --timeout 300 > gpurun_out/pt1.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pt1.log
timeout 300 python bench.py --config c4 --no-e2e --no-cpu > gpurun_out/b_c4.log 2>&1
tail -2 gpurun_out/pt1.log
for f in gpurun_out/b_*.log; do echo $f; python -c "import json,sys; j=json.loads(open('$f').read().strip().splitlines()[-1]); print(j['ms_per_step'], j['roofline']['frac'], j.get('unfused'))"; done
