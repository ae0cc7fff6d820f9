import sys, time, torch
sys.path.insert(0, '.')
import workloads
from tests.planspec import build_gpu_plan
spec = workloads.c4_spec()
plan, ids = build_gpu_plan(spec)
print(plan.explain(ids["g"]))
for n in [1 << 20, 1 << 24, 100_000_000]:
    ins = workloads.c4_inputs(n, device="cuda:0")
    cols, k = plan.run([(n, ins["lineitem"])], ids["g"], 6)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(3):
        plan.run([(n, ins["lineitem"])], ids["g"], 6)
    torch.cuda.synchronize()
    print(n, (time.perf_counter() - t0) / 3 * 1e3, "ms")
