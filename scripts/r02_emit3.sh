#!/bin/bash
O=gpurun_out/r02g; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_scan.py tests/test_gpu_multi.py -q --timeout 300 -x > $O/pytest_scan.log 2>&1; echo "pytest rc=$?" >> $O/pytest_scan.log
tail -2 $O/pytest_scan.log
for a in "" "--dbg 2" "--stages 3" "--variant 3" "--variant 4" "--variant 4 --ctas 2" "--dbg 64"; do
  echo "== $a" >> $O/sweep.log
  timeout 120 python bench.py --config c2 --no-cpu --no-e2e --no-unfused --steps 10 $a 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'): j=json.loads(l); print(j['ms_per_step'], j['roofline']['frac'])
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $O/sweep.log
done
cat $O/sweep.log
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:k_scan_emit -s 2 -c 1 \
    -o $O/prof_c2 -f python bench.py --config c2 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu > $O/ncu_c2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:k_scan_emit -s 2 -c 1 \
