"""GPU parity: fused SELECT / PROJECT / arithmetic chains (k_scan_chain) vs the
oracle, element by element, order included (readings A4, A5, A8)."""
import numpy as np
import pytest

import workloads
from tests.planspec import assert_same, build_gpu_plan, run_gpu, run_oracle

pytestmark = pytest.mark.gpu

DEV = "cuda:0"
# several tiles (2048 rows), ragged tails, empty and single-row inputs
SIZES = [0, 1, 31, 2047, 2048, 2049, 6143, 100_003]


@pytest.mark.parametrize("n", SIZES)
def test_c1_two_selects(n):
    spec = workloads.c1_spec()
    ins = workloads.c1_inputs(n, device=DEV, cfg=0x81)
    got, plan = run_gpu(spec, ins)
    assert_same(got, run_oracle(spec, ins))


@pytest.mark.parametrize("n", SIZES)
@pytest.mark.parametrize("fuse", [True, False])
def test_c2_select_project_select(n, fuse):
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(n, device=DEV, cfg=0x82)
    got, plan = run_gpu(spec, ins, fuse=fuse)
    assert_same(got, run_oracle(spec, ins))
    if fuse and n > 0:
        assert plan.last_launches() == 1        # the whole chain is one kernel


@pytest.mark.parametrize("s", [0.0, 0.1, 0.5, 0.9, 1.0])
def test_selectivity_sweep(s):
    spec = workloads.c2_spec(s, s)
    ins = workloads.c2_inputs(50_000, device=DEV, cfg=0x83)
    got, _ = run_gpu(spec, ins)
    assert_same(got, run_oracle(spec, ins))


@pytest.mark.parametrize("variant", [5, 6, 9])
@pytest.mark.parametrize("n", [1, 6143, 6144, 6145, 300_001])
def test_c2_emit_variants(variant, n):
    """Emitting kernel geometries: 256 x 16, 384 x 8, 384 x 16 (the default for C2;
    48 (group, warp) counters, so the block prefix takes two per lane)."""
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(n, device=DEV, cfg=0x8D)
    got, plan = run_gpu(spec, ins, variant=variant)
    assert_same(got, run_oracle(spec, ins))
    if n > 0:
        assert {5: "k_scan_emit<256,16>", 6: "k_scan_emit<384,8>", 9: "k_scan_emit<384,16>"}[variant] in plan.explain(plan.out_id)


@pytest.mark.parametrize("variant", [7, 8])          # two-team emitting kernels: 2 x 128 x 16, 2 x 256 x 8
@pytest.mark.parametrize("n", SIZES + [300_001])
def test_c2_two_team_kernel(variant, n):
    """Two teams of compute warps on alternate tiles, ring reserved in tile order
    (scan_emit.cu TEAMS = 2): same output, order included."""
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(n, device=DEV, cfg=0x8B)
    got, plan = run_gpu(spec, ins, variant=variant)
    assert_same(got, run_oracle(spec, ins))
    if n > 0:
        assert "2 teams" in plan.explain(plan.out_id)


@pytest.mark.parametrize("variant", [7, 8])
@pytest.mark.parametrize("s", [0.0, 0.1, 0.9, 1.0])
def test_two_team_selectivity(variant, s):
    """All-survive blocks go to the L2 ring, small ones to shared memory: both rings'
    reservations pass between the teams."""
    spec = workloads.c2_spec(s, s)
    ins = workloads.c2_inputs(200_000, device=DEV, cfg=0x8C)
    got, _ = run_gpu(spec, ins, variant=variant)
    assert_same(got, run_oracle(spec, ins))


@pytest.mark.parametrize("stages", [1, 2, 3, 4])
def test_stage_counts(stages):
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(70_001, device=DEV, cfg=0x84)
    got, _ = run_gpu(spec, ins, stages=stages)
    assert_same(got, run_oracle(spec, ins))


def test_unaligned_columns_take_the_plain_load_path():
    import torch
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(40_001, device=DEV, cfg=0x85)
    shifted = {"R": [c[1:] for c in ins["R"]]}          # 4-byte offset: not 16-B aligned
    assert shifted["R"][0].data_ptr() % 16 != 0
    got, _ = run_gpu(spec, shifted)
    assert_same(got, run_oracle(spec, shifted))


def test_deterministic_repeat_and_fused_equals_unfused():
    spec = workloads.c2_spec(0.3, 0.7)
    ins = workloads.c2_inputs(300_000, device=DEV, cfg=0x86)
    a, _ = run_gpu(spec, ins)
    b, _ = run_gpu(spec, ins)
    c, _ = run_gpu(spec, ins, fuse=False)
    assert_same(a, b)
    assert_same(a, c)


def test_arithmetic_types_and_wrap():
    import torch
    rng = np.random.default_rng(3)
    n = 20_011
    cols = [torch.from_numpy(rng.integers(-2**31, 2**31, n, dtype=np.int64).astype(np.int32)).to(DEV),
            torch.from_numpy(rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32).view(np.int32)).to(DEV),
            torch.from_numpy(rng.integers(-2**62, 2**62, n, dtype=np.int64)).to(DEV),
            torch.from_numpy(rng.integers(0, 2**63, n, dtype=np.int64)).to(DEV),
            torch.from_numpy(rng.integers(0, 256, n, dtype=np.int64).astype(np.uint8)).to(DEV)]
    types = ["i32", "u32", "i64", "u64", "u8"]
    exprs = [("col", 0, "i32"), ("col", 1, "u32"), ("col", 2, "i64"), ("col", 3, "u64"), ("col", 4, "u8"),
             ("mul", 0, 0, "i32"),                 # 5 i32 wrap
             ("add", 1, 1, "u32"),                 # 6 u32 wrap
             ("col", 0, "i64"),                    # 7 sign-extend
             ("mul", 2, 7, "i64"),                 # 8 i64 wrap
             ("sub", 3, 2, "u64"),                 # 9 mixed -> u64
             ("divc", 2, -7, "i64"),               # 10 trunc toward zero
             ("const", 5, "i32"), ("sub", 11, 0, "i32"),   # 12: 5 - c0 (reverse subtract)
             ("col", 4, "u32"), ("divc", 13, 3, "u32"),    # 14 u8 -> u32 / 3
             ("col", 1, "i32")]                            # 15 reinterpret u32 bits as i32
    spec = {"inputs": {"R": {"types": types}},
            "nodes": [{"id": "s", "op": "select", "in": "R", "preds": [(4, ">=", 17), (0, "!=", ("col", 0))]},
                      {"id": "s0", "op": "select", "in": "R", "preds": [(4, ">=", 17)]},
                      {"id": "p", "op": "project", "in": "s0", "exprs": exprs,
                       "roots": [5, 6, 8, 9, 10, 12, 14, 15, 4, 11]},
                      {"id": "q", "op": "select", "in": "p", "preds": [(0, ">", -1000), (7, "<", ("col", 0))]}],
            "out": "q"}
    ins = {"R": cols}
    got, _ = run_gpu(spec, ins)
    assert_same(got, run_oracle(spec, ins))


def test_random_chains_against_oracle():
    import torch
    rng = np.random.default_rng(12345)
    for trial in range(25):
        n = int(rng.integers(0, 9000))
        types = [str(t) for t in rng.choice(["i32", "u32", "i64", "u64", "u8"], size=int(rng.integers(1, 6)))]
        info = {"i32": (-2**31, 2**31), "u32": (0, 2**32), "i64": (-2**63, 2**63), "u64": (0, 2**64),
                "u8": (0, 256)}
        cols = []
        for t in types:
            raw = rng.integers(-2**63, 2**63 - 1, n, dtype=np.int64)      # random 64-bit patterns
            if t in ("i64", "u64"):
                a = raw
            elif t in ("i32", "u32"):
                a = raw.astype(np.int32)                                  # keeps the low 32 bits
            else:
                a = (raw & 255).astype(np.uint8)
            cols.append(torch.from_numpy(a).to(DEV))
        nodes, cur, cur_types = [], "R", list(types)
        for k in range(int(rng.integers(1, 5))):
            if rng.random() < 0.6:
                c = int(rng.integers(0, len(cur_types)))
                t = cur_types[c]
                lo, hi = info[t]
                k_const = int(rng.integers(max(lo, -2**62), min(hi, 2**62)))
                op = str(rng.choice(["<", "<=", ">", ">=", "==", "!="]))
                same = [j for j, tt in enumerate(cur_types) if tt == t and j != c]
                rhs = ("col", int(rng.choice(same))) if same and rng.random() < 0.3 else k_const
                nodes.append({"id": f"n{k}", "op": "select", "in": cur, "preds": [(c, op, rhs)]})
            else:
                exprs, roots = [], []
                for j, t in enumerate(cur_types):
                    exprs.append(("col", j, t))
                nout = int(rng.integers(1, 5))
                new_types = []
                for _ in range(nout):
                    a = int(rng.integers(0, len(cur_types)))
                    r = rng.random()
                    if r < 0.4:
                        roots.append(a)
                        new_types.append(cur_types[a])
                    else:
                        t = str(rng.choice(["i32", "u32", "i64", "u64"]))
                        b = int(rng.integers(0, len(cur_types)))
                        opn = str(rng.choice(["add", "sub", "mul"]))
                        exprs.append((opn, a, b, t))
                        roots.append(len(exprs) - 1)
                        new_types.append(t)
                nodes.append({"id": f"n{k}", "op": "project", "in": cur, "exprs": exprs, "roots": roots})
                cur_types = new_types
            cur = f"n{k}"
        spec = {"inputs": {"R": {"types": types}}, "nodes": nodes, "out": cur}
        ins = {"R": cols}
        got, _ = run_gpu(spec, ins)
        assert_same(got, run_oracle(spec, ins))


def test_capacity_error_reports_required_rows():
    import torch
    from paper_conf_micro_wudcy12_b200 import rw
    spec = workloads.c1_spec(0.9999, 0.9999)
    ins = workloads.c1_inputs(5000, device=DEV, cfg=0x87)
    plan, ids = build_gpu_plan(spec)
    outs = [torch.empty(100, dtype=torch.int32, device=DEV) for _ in range(2)]
    with pytest.raises(rw.RwError) as e:
        plan.execute([(5000, ins["R"])], ids["s2"], outs, 100)
    assert e.value.name == "RW_E_CAPACITY"


def test_async_count_to_device():
    import torch
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(123_457, device=DEV, cfg=0x88)
    plan, ids = build_gpu_plan(spec)
    outs = [torch.empty(123_457, dtype=torch.int32, device=DEV) for _ in range(3)]
    n_dev = torch.zeros(1, dtype=torch.int64, device=DEV)
    assert plan.execute([(123_457, ins["R"])], ids["s2"], outs, 123_457, n_dev=n_dev) is None
    torch.cuda.synchronize()
    ref = run_oracle(spec, ins)
    assert int(n_dev.item()) == ref.n


def test_explain_reports_fused_thread_dependence():
    spec = workloads.c2_spec()
    plan, ids = build_gpu_plan(spec)
    txt = plan.explain(ids["s2"])
    assert "thread dependence, fused" in txt
    assert txt.count("group ") == 1
    plan0, ids0 = build_gpu_plan(spec, fuse=False)
    assert plan0.explain(ids0["s2"]).count("group ") == 3


def _long_chain_spec(nproj, per):
    """nproj PROJECT nodes over (i64 x 3), each computing `per` wrapping sums and keeping
    three columns, then a SELECT: too many micro-ops for one fused group when long."""
    nodes, src = [], "R"
    for k in range(nproj):
        ex = [("col", 0, "i64"), ("col", 1, "i64"), ("col", 2, "i64")]
        acc = 1
        for q in range(per):
            ex.append(("add", acc, q % 3, "i64"))
            acc = len(ex) - 1
        nodes.append({"id": f"p{k}", "op": "project", "in": src, "exprs": ex, "roots": [0, acc, 2]})
        src = f"p{k}"
    nodes.append({"id": "s", "op": "select", "in": src, "preds": [(1, "<", 0)]})
    return {"inputs": {"R": {"types": ["i64"] * 3, "nkey_sorted": 0}}, "nodes": nodes, "out": "s"}


@pytest.mark.parametrize("n", [1, 5000, 100_003])
def test_algorithm2_splits_over_budget_groups(n):
    """Algorithm 2: a chain whose fused kernel would exceed the micro-op
    budget is split greedily (longest fitting prefix first), the prefix materialised;
    result identical to the oracle and to operator-at-a-time."""
    import torch
    spec = _long_chain_spec(8, 9)
    g = torch.Generator().manual_seed(n)
    ins = {"R": [torch.randint(-(2**40), 2**40, (n,), dtype=torch.int64, generator=g).to(DEV) for _ in range(3)]}
    ref = run_oracle(spec, ins)
    got, plan = run_gpu(spec, ins, capacity=max(n, 1))
    assert_same(got, ref)
    ex = plan.explain(plan.out_id)
    assert "Algorithm 2" in ex and "group 1" in ex, ex
    got0, _ = run_gpu(spec, ins, capacity=max(n, 1), fuse=False)
    assert_same(got0, ref)


def test_single_operator_over_budget_is_an_error():
    from paper_conf_micro_wudcy12_b200 import rw
    spec = _long_chain_spec(1, 60)
    import torch
    ins = {"R": [torch.zeros(10, dtype=torch.int64, device=DEV) for _ in range(3)]}
    with pytest.raises(rw.RwError) as e:
        run_gpu(spec, ins)
    assert "RW_E_UNSUPPORTED" in str(e.value)
