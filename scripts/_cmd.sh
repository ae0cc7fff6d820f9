mkdir -p gpurun_out
for v in "--dbg 2" "--dbg 1" "--dbg 2 --stages 2" "--dbg 2 --stages 4" ""; do
  echo "== $v" >> gpurun_out/c2var.log
  timeout 300 python bench.py --config c2 --no-e2e --no-cpu --no-unfused $v | python -c "import json,sys; j=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(j['ms_per_step'], j['roofline']['frac'])" >> gpurun_out/c2var.log 2>&1
done
cat gpurun_out/c2var.log
