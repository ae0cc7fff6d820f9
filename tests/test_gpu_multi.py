"""GPU parity of input-dependence fusion (§4.4, Fig. 14(d)):
several SELECT / PROJECT chains over ONE input run as branches of one k_scan_chain
pass (each tile loaded once).  Every branch output is compared with the oracle
element by element, order included, and with the operator-at-a-time path."""
import pytest
import torch

import workloads
from tests.planspec import assert_same, run_gpu_multi, run_oracle_multi

pytestmark = pytest.mark.gpu

DEV = "cuda:0"
SIZES = [0, 1, 31, 2047, 2048, 2049, 6143, 100_003]


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("k", [2, 3, 4])
def test_pattern_d_selects(n, k):
    spec = workloads.cd_spec(0.25, k)
    ins = workloads.cd_inputs(n, device=DEV, cfg=0x86)
    got, plan = run_gpu_multi(spec, ins)
    for g, r in zip(got, run_oracle_multi(spec, ins)):
        assert_same(g, r)
    if n > 0:
        assert plan.last_launches() == 1          # one pass over the shared input


def mixed_spec():
    """Branches of different shapes over one input: a shared SELECT prefix, a PROJECT
    with arithmetic, a branch without any SELECT, and a col-vs-col predicate."""
    return {"inputs": {"R": {"types": ["i32", "u32", "i32", "i32"], "nkey_sorted": 0}},
            "nodes": [
                {"id": "a", "op": "select", "in": "R", "preds": [(0, "<", 0)]},
                {"id": "a1", "op": "select", "in": "a", "preds": [(3, ">=", workloads.thr_i32(0.3))]},
                {"id": "a2", "op": "project", "in": "a",
                 "exprs": [("col", 2, "i64"), ("col", 1, "i64"), ("mul", 0, 1, "i64"), ("col", 3, "i32")],
                 "roots": [2, 3]},
                {"id": "b", "op": "project", "in": "R",
                 "exprs": [("col", 1, "u32"), ("const", 7, "u32"), ("add", 0, 1, "u32")], "roots": [2]},
                {"id": "c", "op": "select", "in": "R", "preds": [(0, "<=", ("col", 2))]}],
            "outs": ["a1", "a2", "b", "c"], "out": "a1"}


@pytest.mark.parametrize("n", [0, 5, 2049, 70_001])
@pytest.mark.parametrize("fuse", [True, False])
def test_mixed_branches(n, fuse):
    spec = mixed_spec()
    ins = workloads.cd_inputs(n, device=DEV, cfg=0x87)
    got, plan = run_gpu_multi(spec, ins, fuse=fuse)
    for g, r in zip(got, run_oracle_multi(spec, ins)):
        assert_same(g, r)
    if n > 0:
        assert plan.last_launches() == (1 if fuse else 6)   # unfused: a, a1 | a, a2 | b | c


@pytest.mark.parametrize("s", [0.0, 1.0])
def test_selectivity_extremes(s):
    spec = workloads.cd_spec(s, 3)
    ins = workloads.cd_inputs(10_000, device=DEV, cfg=0x88)
    got, _ = run_gpu_multi(spec, ins)
    for g, r in zip(got, run_oracle_multi(spec, ins)):
        assert_same(g, r)


def test_unaligned_bases_and_async_counts():
    from tests.planspec import build_gpu_plan
    spec = workloads.cd_spec(0.5, 2)
    ins = workloads.cd_inputs(20_001, device=DEV, cfg=0x89)
    # offset every column by one element: no TMA, per-thread loads of every tile
    big = workloads.cd_inputs(20_002, device=DEV, cfg=0x89)
    shifted = {"R": [c[1:] for c in big["R"]]}
    ref = run_oracle_multi(spec, shifted)
    plan, ids = build_gpu_plan(spec)
    nodes = [ids[o] for o in spec["outs"]]
    cols = [[torch.empty(20_001, dtype=torch.int32, device=DEV) for _ in range(4)] for _ in nodes]
    ndev = [torch.zeros(1, dtype=torch.int64, device=DEV) for _ in nodes]
    assert plan.execute_multi([(20_001, shifted["R"])], nodes, cols, [20_001] * 2, n_devs=ndev) is None
    torch.cuda.synchronize()
    for k, r in enumerate(ref):
        n = int(ndev[k].item())
        assert n == r.n
        for c in range(4):
            assert (cols[k][c][:n].cpu().numpy().view("int32") == r.cols[c]).all()
    del ins


def test_capacity_error():
    from paper_conf_micro_wudcy12_b200 import rw
    from tests.planspec import build_gpu_plan
    spec = workloads.cd_spec(0.5, 2)
    ins = workloads.cd_inputs(10_000, device=DEV, cfg=0x8a)
    plan, ids = build_gpu_plan(spec)
    nodes = [ids[o] for o in spec["outs"]]
    cols = [[torch.empty(10_000, dtype=torch.int32, device=DEV) for _ in range(4)] for _ in nodes]
    with pytest.raises(rw.RwError) as e:
        plan.execute_multi([(10_000, ins["R"])], nodes, cols, [10_000, 100])
    assert e.value.name == "RW_E_CAPACITY"
