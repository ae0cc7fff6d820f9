"""GPU: the multi-GPU kernels on one device — key-range split, stable P-way merge,
aggregate limb export/import — driven through a simulated P-rank exchange, checked
against the oracle on the unsharded relations (order included)."""
import numpy as np
import pytest

import oracle
import workloads
from tests.planspec import assert_same, build_gpu_plan, run_gpu, run_oracle

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def simulated_exchange(backend, shards, types, splitters, packed=False):
    """What exchange_all() does with all_to_all_single, done in-process for P virtual
    ranks: per-column pieces + rw_merge_runs, or (packed) one u64 image per tuple
    (rw_pack_tuples) + rw_merge_packed_runs, as the product path sends them."""
    import torch
    P = len(shards)
    pieces = [[None] * P for _ in range(P)]          # pieces[src][dst] = list of column slices
    for src, cols in enumerate(shards):
        n = int(cols[0].numel())
        b = backend.split(cols[0], types[0], torch.tensor(splitters, dtype=torch.int64, device=DEV)).tolist()
        cuts = [0] + b + [n]
        for dst in range(P):
            pieces[src][dst] = [c[cuts[dst]:cuts[dst + 1]] for c in cols]
    out = []
    for dst in range(P):
        recv = [torch.cat([pieces[src][dst][c] for src in range(P)]) for c in range(len(types))]
        run_off = [0]
        for src in range(P):
            run_off.append(run_off[-1] + int(pieces[src][dst][0].numel()))
        if packed:
            buf = torch.cat([backend.pack(pieces[src][dst], types) for src in range(P)])
            out.append(backend.merge_packed(buf, types, run_off))
        else:
            out.append(backend.merge(recv, types, run_off))
    return out


@pytest.mark.parametrize("packed", [False, True])
@pytest.mark.parametrize("P", [2, 3, 8])
def test_key_range_sharded_three_way_join_equals_single_gpu(P, packed):
    import torch
    from paper_conf_micro_wudcy12_b200 import dist as rd
    n = 20_000
    spec = workloads.c5_spec()
    full = workloads.c5_inputs(n, device=DEV, cfg=0xA1)          # globally sorted relations
    # rank r holds rows [r n/P, (r+1) n/P) of each relation's generation order, locally sorted
    import rwgen
    shards = {k: [] for k in "RST"}
    for r in range(P):
        s, m = rd.row_range(n, r, P)
        part = workloads.c5_inputs(m, key_space=n, start=s, device=DEV, cfg=0xA1)
        for k in "RST":
            shards[k].append(part[k])
    backend = rd.GpuBackend(0)
    keys = [(c[0], "u32") for k in "RST" for c in shards[k]]
    allk = torch.cat([rd.key_values(k, t) for k, t in keys])
    allk, _ = torch.sort(allk)
    spl = [int(allk[(allk.numel() * (r + 1)) // P].item()) for r in range(P - 1)]
    ex = {k: simulated_exchange(backend, shards[k], ["u32", "u32"], spl, packed) for k in "RST"}
    # each virtual rank's range, merged, equals the slice of the globally sorted relation
    for k in "RST":
        cat = [torch.cat([ex[k][r][c] for r in range(P)]) for c in range(2)]
        assert torch.equal(cat[0], full[k][0]) and torch.equal(cat[1], full[k][1])
    outs = []
    for r in range(P):
        ins = {k: ex[k][r] for k in "RST"}
        ref_r = run_oracle(spec, ins)
        got, _ = run_gpu(spec, ins, capacity=max(ref_r.n, 1))
        outs.append(got)
    ref = run_oracle(spec, full)
    merged = oracle.Relation(ref.types, [np.concatenate([o.cols[c] for o in outs]) for c in range(len(ref.types))])
    assert_same(merged, ref)


@pytest.mark.parametrize("op", ["union", "intersect", "difference"])
@pytest.mark.parametrize("P", [2, 3, 8])
def test_key_range_sharded_setop_equals_single_gpu(op, P):
    """Set operators shard like the JOIN: equal tuples share their key,
    so after the key-range exchange every rank's result is the global result's slice
    of its key range; the rank-order concatenation equals the single-GPU result."""
    import torch
    from paper_conf_micro_wudcy12_b200 import dist as rd
    n = 30_000
    spec = workloads.cs_spec(op)
    full = workloads.cs_inputs(n, device=DEV, cfg=0xA5)
    shards = {k: [] for k in "XY"}
    for r in range(P):
        s, m = rd.row_range(n, r, P)
        part = workloads.cs_inputs(m, key_space=n, start=s, device=DEV, cfg=0xA5)
        for k in "XY":
            shards[k].append(part[k])
    backend = rd.GpuBackend(0)
    allk, _ = torch.sort(torch.cat([rd.key_values(c[0], "u32") for k in "XY" for c in shards[k]]))
    spl = [int(allk[(allk.numel() * (r + 1)) // P].item()) for r in range(P - 1)]
    ex = {k: simulated_exchange(backend, shards[k], ["u32", "u32"], spl) for k in "XY"}
    outs = []
    for r in range(P):
        ins = {k: ex[k][r] for k in "XY"}
        got, _ = run_gpu(spec, ins, capacity=2 * n)
        outs.append(got)
    ref = run_oracle(spec, full)
    merged = oracle.Relation(ref.types, [np.concatenate([o.cols[c] for o in outs]) for c in range(2)])
    assert_same(merged, ref)


def test_split_bounds_and_merge_small():
    import torch
    from paper_conf_micro_wudcy12_b200 import dist as rd
    backend = rd.GpuBackend(0)
    keys = torch.tensor([1, 1, 3, 5, 5, 5, 9], dtype=torch.int32, device=DEV)
    spl = torch.tensor([0, 1, 2, 5, 6, 10], dtype=torch.int64, device=DEV)
    assert backend.split(keys, "i32", spl).tolist() == [0, 0, 2, 3, 6, 7]
    a = [torch.tensor([1, 3, 3, 7], dtype=torch.int64, device=DEV), torch.tensor([0, 1, 2, 3], dtype=torch.int32, device=DEV)]
    b = [torch.tensor([0, 3, 8], dtype=torch.int64, device=DEV), torch.tensor([9, 1, 9], dtype=torch.int32, device=DEV)]
    cols = [torch.cat([a[0], b[0]]), torch.cat([a[1], b[1]])]
    m = backend.merge(cols, ["i64", "i32"], [0, 4, 7])
    assert m[0].tolist() == [0, 1, 3, 3, 3, 7, 8]
    assert m[1].tolist() == [9, 0, 1, 1, 2, 3, 9]     # (3,1) twice: run order kept, then (3,2)


@pytest.mark.parametrize("P", [1, 2, 4])
def test_aggregate_limb_combine_equals_single_gpu(P):
    import torch
    from paper_conf_micro_wudcy12_b200 import dist as rd
    n = 300_000
    spec = workloads.c4_spec()
    full = workloads.c4_inputs(n, device=DEV, cfg=0xA2)
    plan, ids = build_gpu_plan(spec)
    node = ids["g"]
    total = None
    for r in range(P):
        s, m = rd.row_range(n, r, P)
        part = workloads.c4_inputs(m, start=s, device=DEV, cfg=0xA2)
        cols, k = plan.run([(m, part["lineitem"])], node, 6)
        limbs = plan.agg_export(node, cols, n_host=k)
        total = limbs.clone() if total is None else total + limbs      # == all_reduce(SUM)
    types = plan.node_schema(node)
    outs = [torch.empty(6, dtype=rd.STORAGE[t], device=DEV) for t in types]
    k = plan.agg_import(node, total, outs, 6)
    got = oracle.Relation(types, [o[:k].cpu().numpy().view(oracle.NP[t]) for o, t in zip(outs, types)])
    assert_same(got, run_oracle(spec, full))
