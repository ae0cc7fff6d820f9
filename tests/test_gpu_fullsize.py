"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(default plan options).  The oracle is run on chunks it finishes in seconds; offsets
of a chunk inside the GPU output come from torch reductions (an implementation
independent of librw), never from the CUDA path:

* C2 (2^29 x 4 i32): first, last and two interior 2^22-row chunks compared element by
  element (order included); total count vs a torch count of the predicate.
* C4 (6e8 lineitem rows): the full aggregate equals the sum of per-chunk oracle
  aggregates (exact additivity of integer sums), all 600M rows covered.
* C3 (2 x 2^26 Zipf-0.5): |J| = sum_k mL(k) mR(k) via torch.unique; three key ranges
  (including the hottest key) compared with the oracle join of the sub-relations.
"""
import numpy as np
import pytest

import oracle
import workloads
from tests.planspec import NPT, assert_same, build_gpu_plan, run_oracle

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
DEV = "cuda:0"
CH = 1 << 22


def _comp(cols):
    """(u32 key, u32 val) rows as one int64 whose order within a key is the val order."""
    import torch
    return ((cols[0].to(torch.int64) & 0xFFFFFFFF) << 32) | (cols[1].to(torch.int64) & 0xFFFFFFFF)


def _greater_counts(Lc, Rc):
    """For every row (k, v) of L: the rows (k, w) of R with w > v (u32 compare)."""
    import torch
    lc, rc = _comp(Lc), torch.sort(_comp(Rc)).values   # relations are sorted on the key only
    pos = torch.searchsorted(rc, lc, right=True)
    end = torch.searchsorted(rc, (lc & ~0xFFFFFFFF) | 0xFFFFFFFF, right=True)
    return end - pos


def _pairs_greater(Lc, Rc) -> int:
    return int(_greater_counts(Lc, Rc).sum().item())


def _host(cols, types, a, b):
    return oracle.Relation(types, [c[a:b].cpu().numpy().view(NPT[t]) for c, t in zip(cols, types)])


def test_c2_full_size_chunks():
    import torch
    n = workloads.C2_ROWS
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(n, device=DEV)
    plan, ids = build_gpu_plan(spec)
    outs = [torch.empty(n, dtype=torch.int32, device=DEV) for _ in range(3)]
    m = plan.execute([(n, ins["R"])], ids["s2"], outs, n)
    R = ins["R"]
    keep = (R[1] < workloads.thr_i32(0.5)) & (R[3] < workloads.thr_i32(0.5))
    assert m == int(keep.sum().item())
    types = ["i32"] * 4
    for a in [0, 123 * CH, 77 * CH + 5, n - CH]:
        b = min(a + CH, n)
        ref = run_oracle(spec, {"R": [c[a:b] for c in R]})
        off = int(keep[:a].sum().item())
        got = oracle.Relation(ref.types, [o[off:off + ref.n].cpu().numpy().view(np.int32) for o in outs])
        assert_same(got, ref)


def test_c4_full_size_additive():
    import torch
    n = workloads.C4_ROWS
    spec = workloads.c4_spec()
    ins = workloads.c4_inputs(n, device=DEV)
    plan, ids = build_gpu_plan(spec)
    got_cols, k = plan.run([(n, ins["lineitem"])], ids["g"], 6)
    types = plan.node_schema(ids["g"])
    got = {}
    for i in range(k):
        g = (int(got_cols[0][i]), int(got_cols[1][i]))
        got[g] = [int(got_cols[2][i])] + [
            (int(got_cols[4 + 2 * q][i].item()) << 64) + (int(got_cols[3 + 2 * q][i].item()) & ((1 << 64) - 1))
            for q in range(5)]
    ref = {}
    big = 1 << 25
    for a in range(0, n, big):
        b = min(a + big, n)
        part = run_oracle(spec, {"lineitem": [c[a:b] for c in ins["lineitem"]]})
        for i in range(part.n):
            g = (int(part.cols[0][i]), int(part.cols[1][i]))
            row = [int(part.cols[2][i])] + [
                int(part.cols[4 + 2 * q][i]) * (1 << 64) + int(part.cols[3 + 2 * q][i]) for q in range(5)]
            acc = ref.setdefault(g, [0] * 6)
            ref[g] = [x + y for x, y in zip(acc, row)]
    assert sorted(got) == sorted(ref)
    for g in ref:
        assert got[g] == ref[g], g
    assert sum(v[0] for v in ref.values()) > 0.98 * n      # ~98.6% of rows pass the date filter


def test_c3_full_size_cardinality_and_key_ranges():
    import torch
    n = workloads.C3_ROWS
    spec = workloads.c3_spec()
    ins = workloads.c3_inputs(n, device=DEV)
    plan, ids = build_gpu_plan(spec)
    cap = 400_000_000
    outs = [torch.empty(cap, dtype=torch.int32, device=DEV) for _ in range(2)]
    m = plan.execute([(n, ins["L"]), (n, ins["R"])], ids["p"], outs, cap)
    lk = ins["L"][0].to(torch.int64) & 0xFFFFFFFF
    rk = ins["R"][0].to(torch.int64) & 0xFFFFFFFF
    ku, cl = torch.unique_consecutive(lk, return_counts=True)
    kv, cr = torch.unique_consecutive(rk, return_counts=True)
    # |L join R| before the SELECT (property): join the plan without the select
    common_l = torch.isin(ku, kv)
    common_r = torch.isin(kv, ku)
    total = int((cl[common_l] * cr[common_r]).sum().item())
    assert total > 0 and m <= total
    # exact output count: for every L row (k, lval) the R rows of key k with rval > lval,
    # by binary search in R's (key, val) order (torch.searchsorted, independent of librw)
    assert m == _pairs_greater(ins["L"], ins["R"])
    okey = outs[0][:m].to(torch.int64) & 0xFFFFFFFF
    assert bool((okey[1:] >= okey[:-1]).all())
    hot = int(ku[torch.argmax(cl * common_l)].item())
    for lo, hi in [(0, 1 << 24), (hot, hot + 1), (3 << 30, (3 << 30) + (1 << 25))]:
        lsel = (lk >= lo) & (lk < hi)
        rsel = (rk >= lo) & (rk < hi)
        sub = {"L": [c[lsel] for c in ins["L"]], "R": [c[rsel] for c in ins["R"]]}
        ref = run_oracle(spec, sub)
        a = int(torch.searchsorted(okey, torch.tensor([lo], device=DEV)).item())
        got = oracle.Relation(ref.types, [o[a:a + ref.n].cpu().numpy().view(np.uint32) for o in outs])
        assert_same(got, ref)
        b = int(torch.searchsorted(okey, torch.tensor([hi], device=DEV)).item())
        assert b - a == ref.n


def test_pattern_d_full_size_chunks():
    """Input-dependence fusion (bench config cd) at 2^29 x 4 i32, 2 branches, in the
    bench launch configuration: per branch the total count vs a torch count of its
    predicate, and the first / an interior / the last 2^22-row input chunk's
    survivors compared with the oracle element by element."""
    import torch
    n = workloads.C2_ROWS
    spec = workloads.cd_spec(0.25, 2)
    ins = workloads.cd_inputs(n, device=DEV)
    plan, ids = build_gpu_plan(spec)
    nodes = [ids[o] for o in spec["outs"]]
    cap = n // 2
    outs = [[torch.empty(cap, dtype=torch.int32, device=DEV) for _ in range(4)] for _ in nodes]
    ms = plan.execute_multi([(n, ins["R"])], nodes, outs, [cap, cap])
    R = ins["R"]
    for b in range(2):
        keep = R[b] < workloads.thr_i32(0.25)
        assert ms[b] == int(keep.sum().item())
        one = {"inputs": spec["inputs"], "nodes": [spec["nodes"][b]], "out": spec["outs"][b]}
        for a in [0, 91 * CH + 3, n - CH]:
            e = min(a + CH, n)
            ref = run_oracle(one, {"R": [c[a:e] for c in R]})
            off = int(keep[:a].sum().item())
            got = oracle.Relation(ref.types, [o[off:off + ref.n].cpu().numpy().view(np.int32) for o in outs[b]])
            assert_same(got, ref)


def test_setop_full_size_key_ranges():
    """Set operators (bench config cs) at 2 x 2^26 tuples: the result restricted to a
    key range equals the oracle on the inputs restricted to that range (tuples are
    whole, so ranges of the sorted key split every operator exactly); ranges at the
    start, the middle and the end.  Row counts vs torch.unique on packed tuples."""
    import torch
    n = 1 << 26
    ins = workloads.cs_inputs(n, device=DEV)
    X, Y = ins["X"], ins["Y"]
    px = (X[0].to(torch.int64) & 0xffffffff) * 4 + X[1].to(torch.int64)
    py = (Y[0].to(torch.int64) & 0xffffffff) * 4 + Y[1].to(torch.int64)
    ux, uy = torch.unique(px), torch.unique(py)
    both = torch.isin(ux, uy)
    expect = {"union": int(torch.unique(torch.cat([ux, uy])).numel()), "intersect": int(both.sum().item()),
              "difference": int((~both).sum().item())}
    for op in ("union", "intersect", "difference"):
        spec = workloads.cs_spec(op)
        plan, ids = build_gpu_plan(spec)
        outs = [torch.empty(2 * n, dtype=torch.int32, device=DEV) for _ in range(2)]
        m = plan.execute([(n, X), (n, Y)], ids["s"], outs, 2 * n)
        assert m == expect[op]
        key = outs[0][:m].to(torch.int64) & 0xffffffff
        for lo, hi in [(0, 1 << 16), (n // 2, n // 2 + (1 << 16)), (n - (1 << 16), n)]:
            xs = (X[0].to(torch.int64) & 0xffffffff)
            ys = (Y[0].to(torch.int64) & 0xffffffff)
            xa, xb = int(torch.searchsorted(xs, lo)), int(torch.searchsorted(xs, hi))
            ya, yb = int(torch.searchsorted(ys, lo)), int(torch.searchsorted(ys, hi))
            ref = run_oracle(spec, {"X": [c[xa:xb] for c in X], "Y": [c[ya:yb] for c in Y]})
            oa, ob = int(torch.searchsorted(key, lo)), int(torch.searchsorted(key, hi))
            got = oracle.Relation(ref.types, [o[oa:ob].cpu().numpy().view(np.uint32) for o in outs])
            assert_same(got, ref)


def test_c5_full_size_count_and_key_ranges():
    """C5 (3 x 2^27 rows per GPU, JOIN -> JOIN -> SELECT(a < c)) in the bench launch
    configuration (the fused 3-input group): the exact output count
    sum over R rows (k, a) of m_S(k) * #{T rows (k, c): c > a} by binary searches, and
    three key ranges compared element by element with the oracle on the sub-relations."""
    import torch
    n = 1 << 27
    spec = workloads.c5_spec()
    ins = workloads.c5_inputs(n, device=DEV)
    plan, ids = build_gpu_plan(spec)
    assert "3 inputs" in plan.explain(ids["s"])
    cap = 3 * n
    outs = [torch.empty(cap, dtype=torch.int32, device=DEV) for _ in range(4)]
    m = plan.execute([(n, ins["R"]), (n, ins["S"]), (n, ins["T"])], ids["s"], outs, cap)
    R, S, T = ins["R"], ins["S"], ins["T"]
    rk = R[0].to(torch.int64) & 0xFFFFFFFF
    sk = S[0].to(torch.int64) & 0xFFFFFFFF
    ms = torch.searchsorted(sk, rk, right=True) - torch.searchsorted(sk, rk)
    expect = int((ms * _greater_counts(R, T)).sum().item())
    assert m == expect and m > 0.1 * n
    okey = outs[0][:m].to(torch.int64) & 0xFFFFFFFF
    assert bool((okey[1:] >= okey[:-1]).all())
    tk = T[0].to(torch.int64) & 0xFFFFFFFF
    for lo, hi in [(0, 1 << 14), (n // 2, n // 2 + (1 << 14)), (n - (1 << 14), n)]:
        sub = {}
        for name, keys in (("R", rk), ("S", sk), ("T", tk)):
            a, b = int(torch.searchsorted(keys, lo)), int(torch.searchsorted(keys, hi))
            sub[name] = [c[a:b] for c in ins[name]]
        ref = run_oracle(spec, sub)
        a = int(torch.searchsorted(okey, torch.tensor([lo], device=DEV)).item())
        b = int(torch.searchsorted(okey, torch.tensor([hi], device=DEV)).item())
        assert b - a == ref.n
        got = oracle.Relation(ref.types, [o[a:b].cpu().numpy().view(np.uint32) for o in outs])
        assert_same(got, ref)


def test_host_streamed_full_size_equals_device_path():
    """rw_plan_execute_host on C2's 2^29 x 4 i32 from pinned host memory with the default
    2^25-row chunks (the e2e bench path): identical, row order included, to the device
    execute (itself chunk-checked against the oracle above), and its first and last
    streamed chunk's survivors equal the oracle on those rows."""
    import torch
    n = workloads.C2_ROWS
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(n, device=DEV)
    plan, ids = build_gpu_plan(spec)
    dev_out = [torch.empty(n // 2, dtype=torch.int32, device=DEV) for _ in range(3)]
    m = plan.execute([(n, ins["R"])], ids["s2"], dev_out, n // 2)
    host_in = [c.cpu().pin_memory() for c in ins["R"]]
    host_out = [torch.empty(n // 2, dtype=torch.int32).pin_memory() for _ in range(3)]
    mh = plan.execute_host([(n, host_in)], ids["s2"], host_out, n // 2)
    assert mh == m
    for h, d in zip(host_out, dev_out):
        assert torch.equal(h[:m], d[:m].cpu())
    C = 1 << 25
    keep = (ins["R"][1] < workloads.thr_i32(0.5)) & (ins["R"][3] < workloads.thr_i32(0.5))
    for a in (0, n - C):
        ref = run_oracle(spec, {"R": [c[a:a + C] for c in ins["R"]]})
        off = int(keep[:a].sum().item())
        got = oracle.Relation(ref.types, [o[off:off + ref.n].numpy().view(np.int32) for o in host_out])
        assert_same(got, ref)
