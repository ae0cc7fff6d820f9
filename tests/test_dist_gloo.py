"""World-size-2 gloo tests (CPU) of the multi-GPU orchestration in dist.py: the same
splitter / all_to_all_single / merge / combine code paths, with a test backend
whose kernels are numpy + oracle (the GPU kernels are covered by test_gpu_dist.py)."""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _np_backend():
    from paper_conf_micro_wudcy12_b200 import dist as rd

    class NumpyBackend(rd.Backend):
        def split(self, keys, key_type, splitters):
            kv = rd.key_values(keys, key_type).numpy()
            return torch.from_numpy(np.searchsorted(kv, splitters.numpy(), side="left").astype(np.int64))

        def pack(self, cols, types):
            # order-preserving u64 image: columns concatenated, first most significant,
            # signed types with the sign bit flipped (python ints, then int64 storage)
            n = int(cols[0].numel())
            img = [0] * n
            for c, t in zip(cols, types):
                w = rd.WIDTH[t] * 8
                vals = c.numpy().astype(np.int64).tolist()
                for i, v in enumerate(vals):
                    u = v & ((1 << w) - 1)
                    if t in ("i32", "i64"):
                        u ^= 1 << (w - 1)
                    img[i] = (img[i] << w) | u if w < 64 else u
            return torch.tensor([x - (1 << 64) if x >= 1 << 63 else x for x in img], dtype=torch.int64)

        def merge_packed(self, packed, types, run_off):
            u = packed.numpy().view(np.uint64)
            order = np.argsort(u, kind="stable")
            srt = [int(x) for x in u[order]]
            cols = []
            shift = sum(rd.WIDTH[t] * 8 for t in types)
            for t in types:
                w = rd.WIDTH[t] * 8
                shift -= w
                vals = []
                for x in srt:
                    f = (x >> shift) & ((1 << w) - 1)
                    if t in ("i32", "i64"):
                        f ^= 1 << (w - 1)
                    if f >= 1 << (w - 1) and t != "u8":
                        f -= 1 << w
                    vals.append(f)
                cols.append(torch.tensor(vals, dtype=rd.STORAGE[t]))
            return cols

        def merge(self, cols, types, run_off):
            # stable lexicographic sort over all columns (library sort; run order kept)
            keys = [rd.key_values(c, t).numpy() for c, t in zip(cols, types)]
            order = np.lexsort(tuple(reversed(keys)), axis=0) if keys[0].size else np.zeros(0, dtype=np.int64)
            return [c[torch.from_numpy(order)] for c in cols]
    return NumpyBackend()


def _worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import workloads
        from paper_conf_micro_wudcy12_b200 import dist as rd
        from tests.planspec import run_oracle
        be = _np_backend()
        # --- key-range sharded JOIN -> JOIN -> SELECT (C5 shape) ---
        n = 6000
        s, m = rd.row_range(n, rank, world)
        local = workloads.c5_inputs(m, key_space=n, start=s, cfg=0xB1)
        schema = {k: ["u32", "u32"] for k in "RST"}
        mine = rd.exchange_all(be, local, schema, world, samples=64)
        out = run_oracle(workloads.c5_spec(), mine)
        res = {"join_rows": [c.tolist() for c in out.cols],
               "ranges": {k: [mine[k][0].min().item() if mine[k][0].numel() else None,
                              mine[k][0].max().item() if mine[k][0].numel() else None] for k in "RST"}}
        # --- key-range sharded set operators (same exchange as the join) ---
        ns = 5000
        ss, ms = rd.row_range(ns, rank, world)
        lset = workloads.cs_inputs(ms, key_space=ns, start=ss, cfg=0xB3)
        mset = rd.exchange_all(be, lset, {"X": ["u32", "u32"], "Y": ["u32", "u32"]}, world, samples=64)
        res["set_rows"] = {op: [c.tolist() for c in run_oracle(workloads.cs_spec(op), mset).cols]
                           for op in ("union", "intersect", "difference")}
        # --- row-sharded aggregate combined with an int64 SUM all-reduce of limbs ---
        n4 = 20000
        s4, m4 = rd.row_range(n4, rank, world)
        ins = workloads.c4_inputs(m4, start=s4, cfg=0xB2)
        agg = run_oracle(workloads.c4_spec(), ins)
        D, L = 6, 1 + 1 + 5 * 4
        limbs = torch.zeros(D * L, dtype=torch.int64)
        for i in range(agg.n):
            g = int(agg.cols[0][i]) * 2 + int(agg.cols[1][i])
            row = [1, int(agg.cols[2][i])]
            for k in range(5):
                v = (int(agg.cols[4 + 2 * k][i]) << 64) + int(agg.cols[3 + 2 * k][i]) & ((1 << 128) - 1)
                row += [(v >> (32 * j)) & 0xFFFFFFFF for j in range(4)]
            limbs[g * L:(g + 1) * L] = torch.tensor(row)
        rd.allreduce_limbs(limbs)
        res["limbs"] = limbs.tolist()
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


def test_world2_gloo_key_range_join_setops_and_aggregate_combine():
    sys.path.insert(0, ROOT)
    import oracle
    import workloads
    from tests.planspec import run_oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=240) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # key ranges are disjoint and ordered by rank
    for k in "RST":
        assert got[0]["ranges"][k][1] is None or got[1]["ranges"][k][0] is None or \
            (got[0]["ranges"][k][1] & 0xFFFFFFFF) < (got[1]["ranges"][k][0] & 0xFFFFFFFF)
    # rank-order concatenation of the sharded join == single-process join (order included)
    ref = run_oracle(workloads.c5_spec(), workloads.c5_inputs(6000, cfg=0xB1))
    for c in range(len(ref.types)):
        cat = got[0]["join_rows"][c] + got[1]["join_rows"][c]
        assert cat == ref.cols[c].tolist()
    # rank-order concatenation of the sharded set operators == single-process result
    for op in ("union", "intersect", "difference"):
        ref = run_oracle(workloads.cs_spec(op), workloads.cs_inputs(5000, cfg=0xB3))
        for c in range(2):
            assert got[0]["set_rows"][op][c] + got[1]["set_rows"][op][c] == ref.cols[c].tolist(), op
    # all-reduced limbs decode to the single-process aggregate
    assert got[0]["limbs"] == got[1]["limbs"]
    full = run_oracle(workloads.c4_spec(), workloads.c4_inputs(20000, cfg=0xB2))
    L = 22
    limbs = got[0]["limbs"]
    for i in range(full.n):
        g = int(full.cols[0][i]) * 2 + int(full.cols[1][i])
        row = limbs[g * L:(g + 1) * L]
        assert row[0] >= 1 and row[1] == int(full.cols[2][i])
        for k in range(5):
            v = sum(row[2 + 4 * k + j] << (32 * j) for j in range(4)) & ((1 << 128) - 1)
            expect = (int(full.cols[4 + 2 * k][i]) << 64) + int(full.cols[3 + 2 * k][i]) & ((1 << 128) - 1)
            assert v == expect
