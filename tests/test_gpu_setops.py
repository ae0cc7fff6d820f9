"""GPU parity of the set operators (Table 1, reading A24):
k_set_op (merge path over whole tuples) vs the oracle, element by element, order
included, across partition boundaries, duplicates inside an input, signed / 64-bit /
multi-column tuples, empty sides, and a downstream SELECT over the result."""
import numpy as np
import pytest
import torch

import oracle
import workloads
from tests.planspec import assert_same, run_gpu, run_oracle

pytestmark = pytest.mark.gpu
DEV = "cuda:0"
OPS = ["union", "intersect", "difference"]


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("n", [0, 1, 7, 2047, 2048, 5000, 100_003])
def test_setop_uniform(op, n):
    spec = workloads.cs_spec(op)
    ins = workloads.cs_inputs(n, device=DEV, cfg=0xb1)
    got, plan = run_gpu(spec, ins, capacity=2 * max(n, 1))
    assert_same(got, run_oracle(spec, ins))


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("nval,ks", [(1, 50), (2, 3000), (4, 1 << 20)])
def test_setop_heavy_duplicates(op, nval, ks):
    """Long runs of equal tuples spanning many 2048-row partitions, few distinct values."""
    spec = workloads.cs_spec(op)
    ins = workloads.cs_inputs(30_000, device=DEV, cfg=0xb2, nval=nval, key_space=ks)
    got, _ = run_gpu(spec, ins, capacity=60_000)
    assert_same(got, run_oracle(spec, ins))


def sorted_rel(rng, n, types, hi):
    cols = [rng.integers(-hi if t.startswith("i") else 0, hi, n).astype(oracle.NP[t]) for t in types]
    order = np.lexsort(cols[::-1])
    return [c[order] for c in cols]


@pytest.mark.parametrize("op", OPS)
@pytest.mark.parametrize("types", [["i32"], ["i64", "u8"], ["u64", "i32", "u32"], ["i32", "i32", "u8", "i64"]])
def test_setop_types(op, types):
    rng = np.random.default_rng(5)
    spec = {"inputs": {"X": {"types": types, "nkey_sorted": len(types)},
                       "Y": {"types": types, "nkey_sorted": len(types)}},
            "nodes": [{"id": "s", "op": op, "left": "X", "right": "Y"}], "out": "s"}
    tdt = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64, "u8": torch.uint8}
    ins = {}
    for name, n in (("X", 9000), ("Y", 7000)):
        ins[name] = [torch.from_numpy(c.view({"i32": np.int32, "u32": np.int32, "i64": np.int64,
                                               "u64": np.int64, "u8": np.uint8}[t]).copy()).to(DEV)
                     for c, t in zip(sorted_rel(rng, n, types, 12), types)]
    got, _ = run_gpu(spec, ins, capacity=16_000)
    assert_same(got, run_oracle(spec, ins))


@pytest.mark.parametrize("op", OPS)
def test_setop_empty_side(op):
    spec = workloads.cs_spec(op)
    full = workloads.cs_inputs(3000, device=DEV, cfg=0xb3)
    for ins in ({"X": full["X"], "Y": [c[:0] for c in full["Y"]]}, {"X": [c[:0] for c in full["X"]], "Y": full["Y"]}):
        got, _ = run_gpu(spec, ins, capacity=6000)
        assert_same(got, run_oracle(spec, ins))


def test_select_over_union():
    spec = workloads.cs_spec("union")
    spec["nodes"].append({"id": "f", "op": "select", "in": "s", "preds": [(1, "<", 2)]})
    spec["out"] = "f"
    ins = workloads.cs_inputs(50_000, device=DEV, cfg=0xb4)
    got, _ = run_gpu(spec, ins, capacity=100_000)
    assert_same(got, run_oracle(spec, ins))


def test_unsorted_and_type_errors():
    from paper_conf_micro_wudcy12_b200 import rw
    p = rw.Plan()
    a = p.add_input(["u32", "u32"], 1)
    b = p.add_input(["u32", "u32"], 2)
    c = p.add_input(["u32", "i32"], 2)
    with pytest.raises(rw.RwError) as e:
        p.add_setop(a, b, "union")
    assert e.value.name == "RW_E_UNSORTED"
    with pytest.raises(rw.RwError) as e:
        p.add_setop(b, c, "intersect")
    assert e.value.name == "RW_E_TYPE"
