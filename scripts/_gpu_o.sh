mkdir -p gpurun_out/o
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/o/pytest.log 2>&1; tail -n 3 gpurun_out/o/pytest.log
OUT=gpurun_out/o STEPS=20 SPECS="--config c2|--config c1|--config c5|--config cs" KNOBS="" bash scripts/knob_sweep.sh > /dev/null 2>&1
python - > gpurun_out/o/explain.txt 2>&1 <<'PY'
import workloads
from tests.planspec import build_gpu_plan
for name, spec in (("c5", workloads.c5_spec()), ("c2", workloads.c2_spec()), ("c3", workloads.c3_spec())):
    plan, ids = build_gpu_plan(spec)
    print(name, plan.explain(ids[spec["out"]]))
PY
cat gpurun_out/o/sweep.log gpurun_out/o/explain.txt
