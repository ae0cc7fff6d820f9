"""Pins for oracle.evaluate, the plan-spec walker (oracle/__init__.py), independent
of it: (1) hand-worked literal results of every workload spec (C1-C5, patterns (c),
(d), set operators) on tiny inputs, each derived by hand from the definitions of
SURVEY §8(c) c1 and the readings of DESIGN.md §2; (2) tests/bruteforce.evaluate_spec,
a second reader of the spec format written with python ints, on seeded random tiny
relations of each workload's shape.  A misread spec field (roots, ("col", j)
right-hand sides, the nkey default, aggregate column order) fails (1)."""
import numpy as np
import pytest

import oracle
import rwgen
import workloads
from tests import bruteforce as bf

NP = {"i32": np.int32, "u32": np.uint32, "i64": np.int64, "u64": np.uint64, "u8": np.uint8}


def rels(spec, rows):
    out = {}
    for name, inp in spec["inputs"].items():
        ts = inp["types"]
        cols = [np.array([r[c] for r in rows[name]], dtype=NP[t]) for c, t in enumerate(ts)]
        out[name] = oracle.Relation(ts, cols)
    return out


def oracle_rows(spec, rows):
    r = oracle.evaluate(spec, rels(spec, rows))
    return r.types, r.rows()


# ---- (1) hand-worked results --------------------------------------------------
def test_c1_literal():
    # thresholds 2^31 on both columns (reading A13, s = 0.5)
    rows = {"R": [(0, 0), (1 << 31, 0), (5, 1 << 31), ((1 << 31) - 1, (1 << 31) - 1)]}
    assert oracle_rows(workloads.c1_spec(), rows) == (["u32", "u32"], [(0, 0), ((1 << 31) - 1, (1 << 31) - 1)])


def test_c2_literal():
    # sigma(c1 < 0) -> pi[c0, c2, c3] -> sigma(#2 < 0)   (reading A14)
    m = -(1 << 31)
    rows = {"R": [(1, -5, 2, -3), (2, 5, 3, -4), (3, -1, 4, 7), (4, m, 5, m)]}
    assert oracle_rows(workloads.c2_spec(), rows) == (["i32"] * 3, [(1, 2, -3), (4, 5, m)])


def test_c3_literal():
    # join -> sigma(lval < rval) -> pi[key, rval]; output (key, lval, rval) (reading A1)
    rows = {"L": [(1, 5), (1, 7), (2, 1)], "R": [(1, 6), (2, 0), (3, 9)]}
    assert oracle_rows(workloads.c3_spec(), rows) == (["u32", "u32"], [(1, 6)])


def test_cc_literal():
    # key SELECTs: L.key < 2^31, R.key >= 2^30 (pattern (c), Fig. 14(c))
    h, q = 1 << 31, 1 << 30
    rows = {"L": [(1, 5), (q + 1, 0), (h, 0)], "R": [(1, 9), (q + 1, 1), (h, 1)]}
    assert oracle_rows(workloads.cc_spec(), rows) == (["u32", "u32"], [(q + 1, 1)])


def test_c5_literal():
    # (R join S) join T -> sigma(a < c): columns (k, a, b, c)
    rows = {"R": [(1, 1), (2, 5)], "S": [(1, 10), (1, 11), (2, 3)], "T": [(1, 0), (2, 9)]}
    assert oracle_rows(workloads.c5_spec(), rows) == (["u32"] * 4, [(2, 5, 3, 9)])


def test_c4_literal_q1():
    D = rwgen.D_1998_09_02
    # (shipdate, qty, price, disc, tax, rf, ls), cents / percent as in DECIMAL(15,2)
    rows = {"lineitem": [(D - 1, 100, 1000, 5, 2, 0, 1), (D + 1, 100, 7, 7, 7, 0, 1),
                         (D, 200, 3000, 0, 8, 0, 1), (D - 10, 50, 500, 10, 0, 2, 0)]}
    types, got = oracle_rows(workloads.c4_spec(), rows)
    assert types == ["u8", "u8", "i64"] + ["u64", "i64"] * 5
    # group (0,1): 2 rows; disc_price 1000*95 + 3000*100; charge 95000*102 + 300000*108
    # group (2,0): 1 row; disc_price 500*90; charge 45000*100
    assert got == [(0, 1, 2, 300, 0, 4000, 0, 395000, 0, 42090000, 0, 5, 0),
                   (2, 0, 1, 50, 0, 500, 0, 45000, 0, 4500000, 0, 10, 0)]


def test_cd_literal_branches():
    t = workloads.thr_i32(0.25)
    spec = workloads.cd_spec(0.25, 2)
    rows = {"R": [(t - 1, t, 0, 0), (t, t - 1, 1, 1), (t - 5, t - 5, 2, 2)]}
    env = oracle.evaluate(spec, rels(spec, rows), keep_all=True)
    assert env["d0"].rows() == [(t - 1, t, 0, 0), (t - 5, t - 5, 2, 2)]
    assert env["d1"].rows() == [(t, t - 1, 1, 1), (t - 5, t - 5, 2, 2)]


@pytest.mark.parametrize("op,expect", [("union", [(1, 0), (1, 1), (2, 0), (3, 0)]),
                                       ("intersect", [(1, 1)]), ("difference", [(1, 0), (2, 0)])])
def test_cs_literal(op, expect):
    rows = {"X": [(1, 0), (1, 1), (1, 1), (2, 0)], "Y": [(1, 1), (3, 0)]}
    assert oracle_rows(workloads.cs_spec(op), rows) == (["u32", "u32"], expect)


# ---- (2) second reader of the spec on random tiny relations --------------------
def rand_rows(rng, types, n, lo, hi, sorted_cols=0):
    rows = [tuple(int(rng.integers(lo, hi)) for _ in types) for _ in range(n)]
    return sorted(rows) if sorted_cols else rows


def shaped_inputs(name, spec, rng):
    if name == "c4":
        D = rwgen.D_1998_09_02
        return {"lineitem": [(int(D + rng.integers(-3, 3)), int(rng.integers(100, 5001)), int(rng.integers(0, 10_495_001)),
                              int(rng.integers(0, 11)), int(rng.integers(0, 9)), int(rng.integers(0, 3)),
                              int(rng.integers(0, 2))) for _ in range(int(rng.integers(0, 40)))]}
    out = {}
    for k, inp in spec["inputs"].items():
        n = int(rng.integers(0, 12))
        if name in ("c1", "c2", "cd"):
            ts = inp["types"]
            lo, hi = (-(1 << 31), 1 << 31) if ts[0] == "i32" else (0, 1 << 32)
            out[k] = rand_rows(rng, ts, n, lo, hi)
        else:   # sorted join / set inputs over a tiny key space (many equal keys)
            # cc: keys on both sides of its key SELECTs' thresholds 2^30 and 2^31
            keys = [5, (1 << 30) + 1, (1 << 30) + 2, (1 << 31) + 3] if name == "cc" else [0, 1, 2, 3]
            rows = [(keys[int(rng.integers(0, 4))], int(rng.integers(0, 4))) for _ in range(n)]
            out[k] = sorted(rows)
    return out


SPECS = {"c1": workloads.c1_spec(), "c2": workloads.c2_spec(), "c3": workloads.c3_spec(), "cc": workloads.cc_spec(),
         "c4": workloads.c4_spec(), "c5": workloads.c5_spec(), "cd": workloads.cd_spec(0.5, 3),
         "cs_union": workloads.cs_spec("union"), "cs_intersect": workloads.cs_spec("intersect"),
         "cs_difference": workloads.cs_spec("difference")}


@pytest.mark.parametrize("name", sorted(SPECS))
def test_evaluate_matches_bruteforce_walker(name):
    spec = SPECS[name]
    rng = np.random.default_rng(0xE7A1 + sum(map(ord, name)))
    nonempty = 0
    for _ in range(60):
        rows = shaped_inputs(name.split("_")[0], spec, rng)
        types, got = oracle_rows(spec, rows)
        etypes, exp = bf.evaluate_spec(spec, rows)
        assert types == etypes
        assert got == exp
        nonempty += bool(exp)
        if "outs" in spec:
            env = oracle.evaluate(spec, rels(spec, rows), keep_all=True)
            for o in spec["outs"]:
                assert env[o].rows() == bf.evaluate_spec(dict(spec, out=o), rows)[1]
    assert nonempty >= 10


def test_evaluate_random_chains_vs_walker():
    """Random SELECT / PROJECT / arithmetic chains (wrap, DIVC, col-vs-col atoms)."""
    rng = np.random.default_rng(77)
    ops = ["<", "<=", ">", ">=", "==", "!="]
    for trial in range(150):
        t = ["i32", "u32", "i64", "u64"][trial % 4]
        lo, hi = {"i32": (-(1 << 31), 1 << 31), "u32": (0, 1 << 32), "i64": (-(1 << 63), 1 << 63),
                  "u64": (0, 1 << 64)}[t]
        rows = {"R": [tuple(int(x) for x in rng.integers(-3, 4, 3, dtype=np.int64)) if rng.random() < 0.5 and t[0] == "i"
                      else tuple(int(rng.integers(lo, hi, dtype=np.int64 if t[0] == "i" else np.uint64)) if t in ("i64", "u64") else int(rng.integers(lo, hi)) for _ in range(3))
                      for _ in range(int(rng.integers(0, 10)))]}
        exprs = [("col", 0, t), ("col", 1, t), ("col", 2, t), ("const", int(rng.integers(-5, 6)), t),
                 (["add", "sub", "mul"][int(rng.integers(0, 3))], 0, 1, t),
                 ("divc", 4, int(rng.choice([-3, -1, 2, 7])), t),
                 (["add", "sub", "mul"][int(rng.integers(0, 3))], 5, 3, t)]
        roots = [int(x) for x in rng.permutation(7)[:3]]
        spec = {"inputs": {"R": {"types": [t] * 3}},
                "nodes": [{"id": "a", "op": "select", "in": "R",
                           "preds": [(0, ops[int(rng.integers(0, 6))], ("col", 1))]},
                          {"id": "p", "op": "project", "in": "a", "exprs": exprs, "roots": roots},
                          {"id": "b", "op": "select", "in": "p",
                           "preds": [(2, ops[int(rng.integers(0, 6))], int(rng.integers(-3, 4)) % (1 << 32))]}],
                "out": "b"}
        got = oracle_rows(spec, rows)
        assert got == bf.evaluate_spec(spec, rows)
