"""Pins for oracle SELECT (oracle.c or_select; Table 1)."""
import json
import os

import numpy as np
import pytest

import oracle
from tests import bruteforce as bf

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table1.json")))


def rel_from_rows(types, rows):
    cols = list(zip(*rows)) if rows else [[] for _ in types]
    return oracle.Relation(types, [np.array(c, dtype=oracle.NP[t]) for t, c in zip(types, cols)])


def test_table1_select_worked_example():
    g = GOLD["select"]
    r = rel_from_rows(g["types"], g["input"])
    out = oracle.select(r, [tuple(p) for p in g["pred"]])
    assert out.rows() == [tuple(x) for x in g["output"]]


def test_exhaustive_small_relations_all_atoms():
    vals = [0, 1, 2]
    atoms = []
    for col in (0, 1):
        for op in bf.OPS:
            for k in vals:
                atoms.append((col, op, k))
            atoms.append((col, op, ("col", 1 - col)))
    n_checked = 0
    for rows in bf.all_relations(3, 2, vals):
        r = rel_from_rows(["u32", "u32"], rows)
        for a in atoms[::3] if len(rows) == 3 else atoms:
            assert oracle.select(r, [a]).rows() == bf.select(rows, [a])
            n_checked += 1
    assert n_checked > 5000


def test_conjunction_equals_composition():
    # P:188 "only one filter operation is added": sigma_p(sigma_q R) == sigma_{p and q} R
    rng = np.random.default_rng(7)
    a = rng.integers(-2**31, 2**31, size=20000, dtype=np.int64).astype(np.int32)
    b = rng.integers(-2**31, 2**31, size=20000, dtype=np.int64).astype(np.int32)
    r = oracle.Relation(["i32", "i32"], [a, b])
    p, q = (0, "<", 0), (1, ">=", 12345)
    two = oracle.select(oracle.select(r, [p]), [q])
    one = oracle.select(r, [p, q])
    assert two.rows() == one.rows()
    # count against numpy's boolean mask (library routine)
    assert one.n == int(np.count_nonzero((a < 0) & (b >= 12345)))
    assert np.array_equal(one.cols[0], a[(a < 0) & (b >= 12345)])


def test_true_false_special_cases():
    r = oracle.Relation(["u32"], [np.arange(100, dtype=np.uint32)])
    assert oracle.select(r, []).rows() == r.rows()
    assert oracle.select(r, [(0, "<", 0)]).n == 0       # u32 < 0 is never true
    assert oracle.select(r, [(0, ">=", 0)]).n == 100


def test_signedness_follows_declared_type():
    bits = np.array([0xFFFFFFFF, 1], dtype=np.uint32)
    as_u = oracle.Relation(["u32"], [bits])
    as_i = oracle.Relation(["i32"], [bits.view(np.int32)])
    assert oracle.select(as_u, [(0, "<", 0x80000000)]).rows() == [(1,)]
    assert oracle.select(as_i, [(0, "<", 0)]).rows() == [(-1,)]
    big = oracle.Relation(["u64"], [np.array([2**63 + 5, 3], dtype=np.uint64)])
    assert oracle.select(big, [(0, ">", 2**62)]).rows() == [(2**63 + 5,)]


def test_empty_input_and_type_mismatch():
    r = oracle.Relation(["i32", "u32"], [np.zeros(0, np.int32), np.zeros(0, np.uint32)])
    assert oracle.select(r, [(0, "==", 1)]).n == 0
    with pytest.raises(oracle.OracleError) as e:
        oracle.select(r, [(0, "==", ("col", 1))])
    assert e.value.code == "type"
