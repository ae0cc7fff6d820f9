"""Test helpers: run a plan spec on the CUDA path (through the C-ABI binding) and
on the oracle, and compare.  Shares only the plain-data spec and the rwgen inputs
between the two sides."""
from __future__ import annotations

from typing import Dict, List

import numpy as np

import oracle

NPT = {"i32": np.int32, "u32": np.uint32, "i64": np.int64, "u64": np.uint64, "u8": np.uint8}


def build_gpu_plan(spec: Dict, **opts):
    from paper_conf_micro_wudcy12_b200 import rw
    plan = rw.Plan(**opts)
    ids = {}
    for name, inp in spec["inputs"].items():
        ids[name] = plan.add_input(inp["types"], inp.get("nkey_sorted", 0), inp.get("lo"), inp.get("hi"))
    for nd in spec["nodes"]:
        op = nd["op"]
        if op == "select":
            ids[nd["id"]] = plan.add_select(ids[nd["in"]], nd["preds"])
        elif op == "project":
            ids[nd["id"]] = plan.add_project(ids[nd["in"]], nd["exprs"], nd["roots"])
        elif op == "join":
            ids[nd["id"]] = plan.add_join(ids[nd["left"]], ids[nd["right"]], nd.get("nkey", 1))
        elif op in ("union", "intersect", "difference"):
            ids[nd["id"]] = plan.add_setop(ids[nd["left"]], ids[nd["right"]], op)
        elif op == "agg":
            ids[nd["id"]] = plan.add_agg(ids[nd["in"]], nd["gcols"], nd["gdomain"], nd["aggs"])
    return plan, ids


def run_gpu(spec: Dict, inputs: Dict[str, List], capacity=None, plan=None, **opts):
    """inputs: name -> list of CUDA tensors.  Returns an oracle.Relation (host copy)."""
    import torch
    if plan is None:
        plan, ids = build_gpu_plan(spec, **opts)
    else:
        plan, ids = plan
    ins = [(int(inputs[k][0].numel()) if inputs[k] else 0, inputs[k]) for k in spec["inputs"]]
    if capacity is None:
        capacity = max([n for n, _ in ins] + [1])
    plan.out_id = ids[spec["out"]]
    cols, n = plan.run(ins, ids[spec["out"]], capacity)
    types = plan.node_schema(ids[spec["out"]])
    torch.cuda.synchronize()
    host = [c.cpu().numpy().view(NPT[t]) for c, t in zip(cols, types)]
    return oracle.Relation(types, host), plan


def run_gpu_multi(spec: Dict, inputs: Dict[str, List], capacity=None, **opts):
    """Every node of spec["outs"] through rw_plan_execute_multi.  Returns ([Relation], plan)."""
    import torch
    plan, ids = build_gpu_plan(spec, **opts)
    ins = [(int(inputs[k][0].numel()) if inputs[k] else 0, inputs[k]) for k in spec["inputs"]]
    nodes = [ids[o] for o in spec["outs"]]
    res = plan.run_multi(ins, nodes, capacity)
    torch.cuda.synchronize()
    rels = []
    for nd, (cols, n) in zip(nodes, res):
        types = plan.node_schema(nd)
        rels.append(oracle.Relation(types, [c.cpu().numpy().view(NPT[t]) for c, t in zip(cols, types)]))
    return rels, plan


def run_oracle_multi(spec: Dict, inputs: Dict[str, List]):
    env = run_oracle(spec, inputs, keep_all=True)
    return [env[o] for o in spec["outs"]]


def run_oracle(spec: Dict, inputs: Dict[str, List], keep_all: bool = False):
    rels = {}
    for name, inp in spec["inputs"].items():
        cols = [(c.cpu().numpy() if hasattr(c, "cpu") else np.asarray(c)).view(NPT[t])
                for c, t in zip(inputs[name], inp["types"])]
        rels[name] = oracle.Relation(inp["types"], cols)
    return oracle.evaluate(spec, rels, keep_all=keep_all)


def assert_same(gpu: "oracle.Relation", ref: "oracle.Relation", ordered: bool = True):
    """Bit-exact comparison; order included unless ordered=False (canonical sort)."""
    assert gpu.types == ref.types, (gpu.types, ref.types)
    assert gpu.n == ref.n, f"row count {gpu.n} != oracle {ref.n}"
    if ordered:
        for c, (a, b) in enumerate(zip(gpu.cols, ref.cols)):
            if not np.array_equal(a, b):
                bad = int(np.nonzero(a != b)[0][0])
                raise AssertionError(f"column {c} differs first at row {bad}: gpu {a[bad]} oracle {b[bad]}")
    else:
        ka = sorted(gpu.rows())
        kb = sorted(ref.rows())
        assert ka == kb
