"""GPU parity of the rebuilt JOIN path (join2.cu) for the shapes SURVEY §8 asks to fuse:
JOIN -> JOIN on the same key (3 inputs, Fig. 14(b)), JOIN -> chain -> AGG (an aggregate
terminal in the expansion), SELECT / PROJECT upstream of a JOIN (pattern (c), Fig. 13),
and two-column keys (nkey = 2).  Every case: bit-exact vs the oracle, order
included, fused and operator-at-a-time."""
import numpy as np
import pytest
import torch

import workloads
from tests.planspec import assert_same, run_gpu, run_oracle

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def sorted_rel(rng, n, kmax, ncols=2, nkey=1, vmax=1000, kt=np.uint32):
    """n rows, leading nkey key columns in [0, kmax), sorted on every column."""
    cols = [rng.integers(0, kmax, n) for _ in range(nkey)] + [rng.integers(0, vmax, n) for _ in range(ncols - nkey)]
    order = np.lexsort(tuple(reversed(cols)))
    out = []
    for c in cols:
        a = np.asarray(c)[order].astype(kt)
        out.append(torch.from_numpy(a.view(np.int32) if kt in (np.uint32, np.int32) else a).to(DEV))
    return out


def two_rel_spec(types_l, types_r, nodes, out, nkey=1):
    return {"inputs": {"L": {"types": types_l, "nkey_sorted": nkey}, "R": {"types": types_r, "nkey_sorted": nkey}},
            "nodes": nodes, "out": out}


@pytest.mark.parametrize("fuse", [True, False])
@pytest.mark.parametrize("n", [0, 1, 5000, 120_000])
def test_join_then_group_by_aggregate(n, fuse):
    """JOIN -> SELECT -> PROJECT -> AGG (6 groups: register terminal) as one group."""
    rng = np.random.default_rng(11 + n)
    L, R = sorted_rel(rng, n, max(n // 3, 1)), sorted_rel(rng, n, max(n // 3, 1))
    spec = two_rel_spec(["u32", "u32"], ["u32", "u32"], [
        {"id": "j", "op": "join", "left": "L", "right": "R", "nkey": 1},
        {"id": "s", "op": "select", "in": "j", "preds": [(1, "<", 700)]},
        {"id": "p", "op": "project", "in": "s", "exprs": [("col", 1, "u32"), ("divc", 0, 167, "u32"),
                                                          ("col", 2, "u32"), ("col", 2, "u64")], "roots": [1, 2, 3]},
        {"id": "g", "op": "agg", "in": "p", "gcols": [0], "gdomain": [6], "aggs": [("count",), ("sum", 2), ("sum", 1)]}],
        "g")
    ins = {"L": L, "R": R}
    got, plan = run_gpu(spec, ins, capacity=6, fuse=fuse)
    assert_same(got, run_oracle(spec, ins))
    if fuse:
        ex = plan.explain(plan.out_id)
        assert "group 1" not in ex and "<agg>" in ex, ex


@pytest.mark.parametrize("n", [3000, 60_000])
def test_join_aggregate_many_groups_and_direct(n):
    """JOIN -> AGG directly (no chain), 64 groups (global-atomic terminal)."""
    rng = np.random.default_rng(5 + n)
    L = sorted_rel(rng, n, max(n // 4, 1), ncols=3, vmax=64)
    R = sorted_rel(rng, n, max(n // 4, 1), ncols=2)
    spec = two_rel_spec(["u32", "u32", "u32"], ["u32", "u32"], [
        {"id": "j", "op": "join", "left": "L", "right": "R", "nkey": 1},
        {"id": "g", "op": "agg", "in": "j", "gcols": [1], "gdomain": [64], "aggs": [("sum", 3), ("count",), ("sum", 2)]}],
        "g")
    ins = {"L": L, "R": R}
    got, plan = run_gpu(spec, ins, capacity=64)
    assert_same(got, run_oracle(spec, ins))
    assert "group 1" not in plan.explain(plan.out_id)


@pytest.mark.parametrize("n", [0, 2000, 40_000])
def test_three_way_join_aggregate(n):
    """JOIN -> JOIN -> SELECT -> AGG: 3-input expansion with the aggregate terminal."""
    spec = workloads.c5_spec()
    spec["nodes"].append({"id": "g", "op": "agg", "in": "s", "gcols": [], "gdomain": [],
                          "aggs": [("count",), ("sum", 1), ("sum", 3)]})
    spec["out"] = "g"
    ins = workloads.c5_inputs(n, device=DEV, cfg=0xA1)
    got, plan = run_gpu(spec, ins, capacity=1)
    assert_same(got, run_oracle(spec, ins))
    ex = plan.explain(plan.out_id)
    assert "3 inputs" in ex and "group 1" not in ex, ex


@pytest.mark.parametrize("fuse", [True, False])
@pytest.mark.parametrize("n", [1, 7000, 90_000])
def test_value_selects_and_projects_upstream_of_join(n, fuse):
    """Pattern (c) with value SELECTs and an arithmetic, key-preserving PROJECT on the
    inputs (Fig. 13): all fused into the expansion (one group)."""
    rng = np.random.default_rng(100 + n)
    L = sorted_rel(rng, n, max(n // 2, 1), ncols=3)
    R = sorted_rel(rng, n, max(n // 2, 1), ncols=3)
    spec = two_rel_spec(["u32", "u32", "u32"], ["u32", "u32", "u32"], [
        {"id": "fl", "op": "select", "in": "L", "preds": [(1, "<", 600), (2, ">=", ("col", 1))]},
        {"id": "pl", "op": "project", "in": "fl", "exprs": [("col", 0, "u32"), ("col", 1, "u32"), ("col", 2, "u32"),
                                                           ("add", 1, 2, "u32")], "roots": [0, 3, 1]},
        {"id": "fr", "op": "select", "in": "R", "preds": [(2, "!=", 3)]},
        {"id": "j", "op": "join", "left": "pl", "right": "fr", "nkey": 1},
        {"id": "s", "op": "select", "in": "j", "preds": [(1, ">", ("col", 3))]},
        {"id": "p", "op": "project", "in": "s", "exprs": [("col", 0, "u32"), ("col", 1, "u32"), ("col", 4, "u32")],
         "roots": [0, 1, 2]}], "p")
    ins = {"L": L, "R": R}
    ref = run_oracle(spec, ins)
    got, plan = run_gpu(spec, ins, capacity=max(ref.n, 1), fuse=fuse)
    assert_same(got, ref)
    if fuse:
        ex = plan.explain(plan.out_id)
        assert "group 1" not in ex and ex.count("fused into the expansion") == 3, ex


@pytest.mark.parametrize("kt,types", [(np.uint32, ["u32", "u32", "u32"]), (np.int32, ["i32", "i32", "i32"])])
@pytest.mark.parametrize("n", [0, 3000, 80_000])
def test_two_column_keys(n, kt, types):
    """nkey = 2 (P:196 'one JOIN may use the first 2 attributes as a key'): lexicographic
    composite key; output (k0, k1, L rest, R rest) in (key, L row, R row) order."""
    rng = np.random.default_rng(7 + n)
    def rel():
        k0 = rng.integers(-20 if kt == np.int32 else 0, 40, n)
        k1 = rng.integers(-5 if kt == np.int32 else 0, 9, n)
        v = rng.integers(0, 1000, n)
        o = np.lexsort((v, k1, k0))
        return [torch.from_numpy(np.asarray(c)[o].astype(kt).view(np.int32)).to(DEV) for c in (k0, k1, v)]
    spec = two_rel_spec(types, types, [{"id": "j", "op": "join", "left": "L", "right": "R", "nkey": 2},
                                      {"id": "s", "op": "select", "in": "j", "preds": [(2, "<", ("col", 3))]}], "s", nkey=2)
    ins = {"L": rel(), "R": rel()}
    ref = run_oracle(spec, ins)
    got, _ = run_gpu(spec, ins, capacity=max(ref.n, 1))
    assert_same(got, ref)


def test_two_column_keys_three_way():
    rng = np.random.default_rng(99)
    n = 20_000
    def rel():
        k0, k1, v = rng.integers(0, 30, n), rng.integers(0, 6, n), rng.integers(0, 100, n)
        o = np.lexsort((v, k1, k0))
        return [torch.from_numpy(np.asarray(c)[o].astype(np.uint32).view(np.int32)).to(DEV) for c in (k0, k1, v)]
    t = ["u32", "u32", "u32"]
    spec = {"inputs": {"A": {"types": t, "nkey_sorted": 2}, "B": {"types": t, "nkey_sorted": 2},
                       "C": {"types": t, "nkey_sorted": 2}},
            "nodes": [{"id": "ab", "op": "join", "left": "A", "right": "B", "nkey": 2},
                      {"id": "abc", "op": "join", "left": "ab", "right": "C", "nkey": 2},
                      {"id": "s", "op": "select", "in": "abc", "preds": [(2, "<", ("col", 4))]}], "out": "s"}
    ins = {"A": rel(), "B": rel(), "C": rel()}
    ref = run_oracle(spec, ins)
    got, plan = run_gpu(spec, ins, capacity=max(ref.n, 1))
    assert_same(got, ref)
    assert "3 inputs" in plan.explain(plan.out_id)


def test_join_join_fused_explain():
    """Fig. 14(b): the inner JOIN -> outer JOIN edge is CTA dependence, fused."""
    spec = workloads.c5_spec()
    ins = workloads.c5_inputs(1000, device=DEV, cfg=0xA2)
    got, plan = run_gpu(spec, ins, capacity=10_000)
    ex = plan.explain(plan.out_id)
    assert "(JOIN) -> 4(JOIN): CTA dependence, fused" in ex or "(JOIN): CTA dependence, fused" in ex, ex
