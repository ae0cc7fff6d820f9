"""GPU parity: group-by aggregate (Q1, k_scan_chain<agg> + k_agg_finalize) and the
merge-path JOIN (k_join_runs + k_join_expand) fused with downstream operators."""
import numpy as np
import pytest

import oracle
import workloads
from tests.planspec import assert_same, build_gpu_plan, run_gpu, run_oracle

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


@pytest.mark.parametrize("n", [0, 1, 2047, 2049, 100_003, 1_000_000])
@pytest.mark.parametrize("fuse", [True, False])
def test_q1_aggregate(n, fuse):
    spec = workloads.c4_spec()
    ins = workloads.c4_inputs(n, device=DEV, cfg=0x91)
    got, plan = run_gpu(spec, ins, capacity=6, fuse=fuse)
    assert_same(got, run_oracle(spec, ins))


@pytest.mark.parametrize("agg_mode", [0, 1])
def test_q1_both_agg_terminals(agg_mode):
    """agg_mode 0: auto (register one-hot terminal for Q1); 1: thread-private partials."""
    spec = workloads.c4_spec()
    ins = workloads.c4_inputs(300_001, device=DEV, cfg=0x93)
    got, plan = run_gpu(spec, ins, capacity=6, agg_mode=agg_mode)
    assert_same(got, run_oracle(spec, ins))
    want = "partial flush every" if agg_mode == 1 else "register one-hot"
    assert want in plan.explain(plan.out_id)


@pytest.mark.parametrize("agg_mode", [0, 2])
@pytest.mark.parametrize("n", [1, 2303, 2305, 300_001])
def test_q1_fused_row_path_and_interpreter(agg_mode, n):
    """The Q1 program shape runs fused per row in the 576-thread instance (agg_mode 0),
    or through the micro-op interpreter (agg_mode 2): both equal the oracle."""
    spec = workloads.c4_spec()
    ins = workloads.c4_inputs(n, device=DEV, cfg=0x96)
    got, plan = run_gpu(spec, ins, capacity=6, agg_mode=agg_mode)
    assert_same(got, run_oracle(spec, ins))
    assert ("Q1 program fused per row" in plan.explain(plan.out_id)) == (agg_mode == 0)


@pytest.mark.parametrize("variant", [4, 5, 1, 6, 0])
@pytest.mark.parametrize("n", [1, 1919, 1921, 300_001])
def test_q1_wide_cta_variants(variant, n):
    """384 x 5 / 448 x 4 / 256 x 8 / 480 x 4 / 544 x 4 (default for Q1's 5 sums with 2
    narrow ones, 32-bit partials) compute threads (aggregate kernels carry no writer
    warps): tiles of 1920 / 1792 / 2048 / 1920 / 2176 rows, ragged tails."""
    spec = workloads.c4_spec()
    ins = workloads.c4_inputs(n, device=DEV, cfg=0x94)
    got, plan = run_gpu(spec, ins, capacity=6, variant=variant)
    assert_same(got, run_oracle(spec, ins))
    assert {4: "tile 1920", 5: "tile 1792", 1: "tile 2048", 6: "tile 1920 rows (4/thread)",
            0: "tile 2304 rows (4/thread)"}[variant] in plan.explain(plan.out_id)


@pytest.mark.parametrize("lo,hi", [(-1000, 1000), (-(2**40), 2**40), (-(2**63), 2**63 - 1), (5, 5)])
@pytest.mark.parametrize("D", [1, 7, 64])
def test_warp_agg_signed_bounds_and_many_groups(lo, hi, D):
    """Signed sums whose declared bounds give 1, 2 and 3 27-bit chunks (value - lo),
    and up to 64 groups (every batch of 32 rows visits many distinct groups)."""
    import torch
    n = 70_001
    gen = torch.Generator().manual_seed(D * 7 + (hi & 0xff))
    v = torch.randint(lo, hi + 1, (n,), dtype=torch.int64, generator=gen) if hi < 2**63 - 1 else \
        torch.randint(-(2**63), 2**63 - 1, (n,), dtype=torch.int64, generator=gen)
    v[:3] = torch.tensor([lo, hi, lo])
    w = torch.randint(-(2**31), 2**31 - 1, (n,), dtype=torch.int64, generator=gen).to(torch.int32)
    g = torch.randint(0, D, (n,), dtype=torch.int64, generator=gen).to(torch.uint8)
    spec = {"inputs": {"R": {"types": ["u8", "i64", "i32"], "lo": [0, lo, -(2**31)], "hi": [D - 1, hi, 2**31 - 1]}},
            "nodes": [{"id": "a", "op": "agg", "in": "R", "gcols": [0], "gdomain": [D],
                       "aggs": [("sum", 1), ("count",), ("sum", 2), ("sum", 1)]}], "out": "a"}
    ins = {"R": [g.to(DEV), v.to(DEV), w.to(DEV)]}
    got, plan = run_gpu(spec, ins, capacity=D)
    assert ("register one-hot" in plan.explain(plan.out_id)) == (D <= 6 and lo >= -(2**40))
    assert_same(got, run_oracle(spec, ins))


def test_q1_without_bounds_flushes_every_row():
    spec = workloads.c4_spec()
    spec["inputs"]["lineitem"] = {"types": workloads.Q1_TYPES}          # no declared bounds
    ins = workloads.c4_inputs(60_000, device=DEV, cfg=0x92)
    got, _ = run_gpu(spec, ins, capacity=6)
    assert_same(got, run_oracle(spec, ins))


def test_sum_beyond_int64_is_exact():
    import torch
    n = 50_000
    v = torch.full((n,), 2**62 + 7, dtype=torch.int64, device=DEV)
    g = (torch.arange(n, device=DEV) % 3).to(torch.uint8)
    u = torch.full((n,), -1, dtype=torch.int64, device=DEV)              # u64 max
    spec = {"inputs": {"R": {"types": ["u8", "i64", "u64"]}},
            "nodes": [{"id": "a", "op": "agg", "in": "R", "gcols": [0], "gdomain": [3],
                       "aggs": [("sum", 1), ("count",), ("sum", 2)]}], "out": "a"}
    ins = {"R": [g, v, u]}
    got, _ = run_gpu(spec, ins, capacity=3)
    ref = run_oracle(spec, ins)
    assert_same(got, ref)
    assert oracle.sum128(got.cols[1], got.cols[2])[0] == 16667 * (2**62 + 7)


def test_agg_domain_error():
    import torch
    from paper_conf_micro_wudcy12_b200 import rw
    g = torch.tensor([0, 1, 7], dtype=torch.uint8, device=DEV)
    spec = {"inputs": {"R": {"types": ["u8"]}},
            "nodes": [{"id": "a", "op": "agg", "in": "R", "gcols": [0], "gdomain": [3], "aggs": [("count",)]}],
            "out": "a"}
    with pytest.raises(rw.RwError) as e:
        run_gpu(spec, {"R": [g]}, capacity=3)
    assert e.value.name == "RW_E_DOMAIN"


@pytest.mark.parametrize("n", [0, 1, 100, 5000, 200_000])
@pytest.mark.parametrize("fuse", [True, False])
def test_c3_zipf_join_select_project(n, fuse):
    spec = workloads.c3_spec()
    ins = workloads.c3_inputs(n, device=DEV, cfg=0x93)
    ref = run_oracle(spec, ins)
    got, _ = run_gpu(spec, ins, capacity=max(ref.n, 1), fuse=fuse)
    assert_same(got, ref)


def test_join_hot_key_spans_many_tiles():
    import torch
    # one key with 3000 x 2000 matches (6M candidates, > 2600 expansion tiles) plus noise
    lk = torch.cat([torch.arange(0, 500, device=DEV), torch.full((3000,), 777, device=DEV),
                    torch.arange(1000, 1500, device=DEV)]).to(torch.int32)
    rk = torch.cat([torch.arange(0, 800, 2, device=DEV), torch.full((2000,), 777, device=DEV),
                    torch.arange(1000, 3000, 3, device=DEV)]).to(torch.int32)
    lv = torch.arange(lk.numel(), device=DEV, dtype=torch.int32) * 7
    rv = torch.arange(rk.numel(), device=DEV, dtype=torch.int32) * 5 + 3
    lk, _ = torch.sort(lk)
    rk, _ = torch.sort(rk)
    spec = workloads.c3_spec()
    ins = {"L": [lk, lv], "R": [rk, rv]}
    ref = run_oracle(spec, ins)
    got, _ = run_gpu(spec, ins, capacity=ref.n)
    assert_same(got, ref)


def test_join_signed_and_64bit_keys():
    import torch
    rng = np.random.default_rng(4)
    for kt, st in (("i32", np.int32), ("i64", np.int64), ("u64", np.int64)):
        a = np.sort(rng.integers(-50, 50, 3000).astype(st)) if kt != "u64" else \
            np.sort(rng.integers(0, 100, 3000).astype(np.uint64)).view(np.int64)
        b = np.sort(rng.integers(-50, 50, 2500).astype(st)) if kt != "u64" else \
            np.sort(rng.integers(0, 100, 2500).astype(np.uint64)).view(np.int64)
        spec = {"inputs": {"L": {"types": [kt, "u8"], "nkey_sorted": 1},
                           "R": {"types": [kt, "i64", "u32"], "nkey_sorted": 1}},
                "nodes": [{"id": "j", "op": "join", "left": "L", "right": "R", "nkey": 1}], "out": "j"}
        ins = {"L": [torch.from_numpy(a).to(DEV), torch.from_numpy((np.arange(3000) % 251).astype(np.uint8)).to(DEV)],
               "R": [torch.from_numpy(b).to(DEV), torch.from_numpy(np.arange(2500, dtype=np.int64) * -3).to(DEV),
                     torch.from_numpy(np.arange(2500, dtype=np.int32)).to(DEV)]}
        ref = run_oracle(spec, ins)
        got, _ = run_gpu(spec, ins, capacity=ref.n)
        assert_same(got, ref)


@pytest.mark.parametrize("n", [0, 1000, 30_000])
def test_c5_three_way_join(n):
    spec = workloads.c5_spec()
    ins = workloads.c5_inputs(n, device=DEV, cfg=0x94)
    ref = run_oracle(spec, ins)
    got, _ = run_gpu(spec, ins, capacity=max(ref.n, 1))
    assert_same(got, ref)


def test_join_then_aggregate():
    spec = workloads.c3_spec()
    spec["nodes"].append({"id": "g", "op": "agg", "in": "p", "gcols": [], "gdomain": [],
                          "aggs": [("count",), ("sum", 1)]})
    spec["out"] = "g"
    ins = workloads.c3_inputs(20_000, device=DEV, cfg=0x95)
    got, _ = run_gpu(spec, ins, capacity=1)
    assert_same(got, run_oracle(spec, ins))


def test_pattern_c_selects_upstream_of_join():
    """Fig. 14(c) shape: SELECTs on both JOIN inputs, then the join and a
    downstream SELECT + PROJECT.  The upstream value SELECTs are fused into the join's
    expansion (N2, Fig. 13): one kernel group."""
    spec = workloads.c3_spec()
    spec["nodes"] = [{"id": "fl", "op": "select", "in": "L", "preds": [(1, "<", workloads.thr_u32(0.6))]},
                     {"id": "fr", "op": "select", "in": "R", "preds": [(1, ">=", workloads.thr_u32(0.3))]},
                     {"id": "j", "op": "join", "left": "fl", "right": "fr", "nkey": 1}] + spec["nodes"][1:]
    ins = workloads.c3_inputs(30_000, device=DEV, cfg=0x96)
    got, plan = run_gpu(spec, ins, capacity=400_000)
    assert_same(got, run_oracle(spec, ins))
    ex = plan.explain(plan.out_id)
    assert "group 1" not in ex and ex.count("fused into the expansion") == 2, ex


@pytest.mark.parametrize("n", [0, 1000, 30_000, 200_000])
@pytest.mark.parametrize("fuse", [True, False])
def test_n2_key_selects_fused_into_join(n, fuse):
    """SELECTs on the join key upstream of both JOIN inputs (pattern (c), Fig. 13,
    SURVEY §8(f) N2): fused into the run matching (whole key runs kept or dropped), the
    join reads the unfiltered relations; no SELECT kernel runs.  Bit-exact vs oracle."""
    spec = workloads.c3_spec()
    k1, k2, k3 = workloads.thr_u32(0.7), workloads.thr_u32(0.2), workloads.thr_u32(0.5)
    spec["nodes"] = [{"id": "fl", "op": "select", "in": "L", "preds": [(0, "<", k1)]},
                     {"id": "fl2", "op": "select", "in": "fl", "preds": [(0, "!=", k3)]},
                     {"id": "fr", "op": "select", "in": "R", "preds": [(0, ">=", k2), (0, "<=", k1 + 12345)]},
                     {"id": "j", "op": "join", "left": "fl2", "right": "fr", "nkey": 1}] + spec["nodes"][1:]
    ins = workloads.c3_inputs(n, device=DEV, cfg=0x97)
    got, plan = run_gpu(spec, ins, capacity=8 * max(n, 1) + 1024, fuse=fuse)
    assert_same(got, run_oracle(spec, ins))
    ex = plan.explain(plan.out_id)
    if fuse:
        assert ex.count("key SELECT") == 3 and "group 1" not in ex, ex


def test_n2_mixed_key_and_value_selects():
    """A key SELECT on L is fused into the run matching; a value SELECT on R is fused into
    the expansion (evaluated on the gathered R row of every candidate): one group."""
    spec = workloads.c3_spec()
    spec["nodes"] = [{"id": "fl", "op": "select", "in": "L", "preds": [(0, ">", workloads.thr_u32(0.1))]},
                     {"id": "fr", "op": "select", "in": "R", "preds": [(1, "<", workloads.thr_u32(0.5))]},
                     {"id": "j", "op": "join", "left": "fl", "right": "fr", "nkey": 1}] + spec["nodes"][1:]
    ins = workloads.c3_inputs(50_000, device=DEV, cfg=0x98)
    got, plan = run_gpu(spec, ins, capacity=500_000)
    assert_same(got, run_oracle(spec, ins))
    ex = plan.explain(plan.out_id)
    assert ex.count("key SELECT") == 1 and "group 1" not in ex and "upstream of the join, input 1" in ex, ex


def test_n2_signed_keys():
    import torch
    rng = np.random.default_rng(3)
    def rel(n):
        k = np.sort(rng.integers(-500, 500, n)).astype(np.int32)
        v = rng.integers(0, 1000, n).astype(np.int32)
        o = np.lexsort((v, k))
        return [torch.from_numpy(k[o].copy()).to(DEV), torch.from_numpy(v[o].copy()).to(DEV)]
    spec = {"inputs": {"L": {"types": ["i32", "i32"], "nkey_sorted": 1}, "R": {"types": ["i32", "i32"], "nkey_sorted": 1}},
            "nodes": [{"id": "fl", "op": "select", "in": "L", "preds": [(0, ">=", -100), (0, "<", 250)]},
                      {"id": "j", "op": "join", "left": "fl", "right": "R", "nkey": 1}],
            "out": "j"}
    ins = {"L": rel(20_000), "R": rel(15_000)}
    got, plan = run_gpu(spec, ins, capacity=2_000_000)
    assert_same(got, run_oracle(spec, ins))
    assert "key SELECT" in plan.explain(plan.out_id)


def test_q1_declared_bound_violation_is_reported():
    """A summed narrow column (disc, declared in [0, 10]) holding a value outside its
    declared bounds: the 32-bit partials could be inexact, so the execute reports
    RW_E_DOMAIN instead of returning silently wrong sums (rw.h, rw_plan_add_input)."""
    from paper_conf_micro_wudcy12_b200 import rw
    spec = workloads.c4_spec()
    ins = workloads.c4_inputs(50_001, device=DEV, cfg=0x95)
    import rwgen
    ins["lineitem"][0][12345] = rwgen.D_1998_09_02 - 10   # passes the SELECT
    ins["lineitem"][3][12345] = 70_000        # disc far above its declared hi = 10 (and above 2^16)
    with pytest.raises(rw.RwError) as e:
        run_gpu(spec, ins, capacity=6)
    assert "declared" in str(e.value)
    # the same data with the bound not declared narrow: exact, no error
    spec2 = workloads.c4_spec()
    spec2["inputs"]["lineitem"]["hi"] = list(spec2["inputs"]["lineitem"]["hi"])
    spec2["inputs"]["lineitem"]["hi"][3] = 1 << 40
    got, _ = run_gpu(spec2, ins, capacity=6)
    assert_same(got, run_oracle(spec2, ins))
