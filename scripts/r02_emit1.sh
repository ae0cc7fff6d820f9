#!/bin/bash
# emitting scan kernel: parity of the scan paths, then C2 / cd bench lines and a knob sweep
O=gpurun_out/r02b; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_scan.py tests/test_gpu_multi.py tests/test_gpu_literal.py tests/test_gpu_host_stream.py -q --timeout 300 -x > $O/pytest_scan.log 2>&1; echo "pytest rc=$?" >> $O/pytest_scan.log
tail -3 $O/pytest_scan.log
timeout 300 python bench.py --config c2 --no-cpu --no-e2e > $O/bench_c2.log 2>&1
for a in "--ctas 1 --stages 6" "--ctas 1 --stages 5" "--ctas 1 --stages 7" "--ctas 2 --stages 3 --items 4" "--ctas 2 --stages 6 --items 4" "--variant 3" "--defer 1" "--defer 2" "--defer 5"; do
  echo "== $a" >> $O/sweep.log
  timeout 120 python bench.py --config c2 --no-cpu --no-e2e --no-unfused --steps 10 $a 2>&1 | python -c "import json,sys
for l in sys.stdin:
  if l.startswith('{'): j=json.loads(l); print(j['ms_per_step'], j['roofline']['frac'])
  elif 'Error' in l or 'error' in l: print(l.strip())" >> $O/sweep.log
done
timeout 300 python bench.py --config cd --no-cpu --no-e2e > $O/bench_cd.log 2>&1
timeout 300 python bench.py --config c1 --no-cpu --no-e2e > $O/bench_c1.log 2>&1
cat $O/sweep.log
