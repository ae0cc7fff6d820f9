"""Diagnostic: per-tile phase timestamps of the C2 scan kernel (dbg=4)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads
from tests.planspec import build_gpu_plan

def main(stages, ctas, ring, extra=0, cfg="c2"):
    if cfg == "c3":
        rows = 1 << 26
        spec = workloads.c3_spec()
        ins = workloads.c3_inputs(rows, device="cuda:0")
    elif cfg == "c4":
        rows = 600_000_000
        spec = workloads.c4_spec()
        ins = workloads.c4_inputs(rows, 0, "cuda:0")
    else:
        rows = 1 << 29
        spec = workloads.c2_spec()
        ins = workloads.c2_inputs(rows, 0, "cuda:0")
    T = {"c4": 1792, "c3": 2304}.get(cfg, 2048)
    nt = (rows + T - 1) // T if cfg != "c3" else (400_000_000 + T - 1) // T
    ts = torch.zeros(nt * 12, dtype=torch.int64, device="cuda:0")
    plan, ids = build_gpu_plan(spec, stages=stages, ctas_per_sm=ctas, defer=ring, dbg=4 | extra, dbg_ts=ts.data_ptr())
    out_node = ids[spec["out"]]
    types = plan.node_schema(out_node)
    dt = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64, "u8": torch.uint8}
    cap = {"c4": 6, "c3": 400_000_000}.get(cfg, rows)
    outs = [torch.empty(cap, dtype=dt[t], device="cuda:0") for t in types]
    nd = torch.zeros(1, dtype=torch.int64, device="cuda:0")
    print(plan.explain(out_node))
    for _ in range(3):
        plan.execute([(rows, ins[k]) for k in spec["inputs"]], out_node, outs, cap, n_dev=nd)
    torch.cuda.synchronize()
    a = ts.view(nt, 12).double()
    if cfg == "c3":
        nt = int((a[:, 0] > 0).sum())
        a = a[:nt]
    t0 = a[:, 0].min()
    d = {"load(claim->data)": a[:, 1] - a[:, 0], "ops(data->ops)": a[:, 6] - a[:, 1], "ballot(ops->bar1)": a[:, 7] - a[:, 6], "scan(bar1->agg)": a[:, 2] - a[:, 7],
         "reserve(agg->reserved)": a[:, 9] - a[:, 2], "ring wait+scatter(->arrived)": a[:, 8] - a[:, 9], "writer queue(arrived->wstart)": a[:, 5] - a[:, 8], "lookback(wstart->offset)": a[:, 3] - a[:, 5], "store(offset->stored)": a[:, 4] - a[:, 3],
         "total(claim->stored)": a[:, 4] - a[:, 0]}
    if cfg == "c3":
        d["fill: records(data->cached)"] = a[:, 10] - a[:, 1]
        d["fill: search+gather(cached->gathered)"] = a[:, 11] - a[:, 10]
        d["fill->ops"] = a[:, 6] - a[:, 11]
    if cfg == "c4":
        a[:, 3] = a[:, 2]; a[:, 4] = a[:, 2]; a[:, 5] = a[:, 2]; a[:, 7] = a[:, 6]
    res = {"cfg": [stages, ctas, ring, extra, cfg], "kernel_us": float((a[:, 4].max() - t0) / 1e3)}
    for k, v in d.items():
        q = torch.quantile(v[: min(nt, 1 << 24)] / 1e3, torch.tensor([0.1, 0.5, 0.9, 0.99], dtype=torch.float64, device=v.device))
        res[k] = [round(float(x), 2) for x in q]
    print(json.dumps(res))

if __name__ == "__main__":
    main(*[int(x) for x in sys.argv[1:5]], *sys.argv[5:6])
