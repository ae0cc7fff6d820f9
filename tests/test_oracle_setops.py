"""Pins for the oracle set operators (oracle.c or_setop; Table 1, reading A24:
whole-tuple membership, set semantics, inputs sorted on every attribute, ascending
output).  Checked against the paper's worked examples, Python's own hash sets on
every small relation, numpy.unique at scale, and the algebra of sets."""
import json
import os
from itertools import product

import numpy as np
import pytest

import oracle
from tests.test_oracle_select import rel_from_rows

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table1.json")))
PY = {"union": lambda a, b: a | b, "intersect": lambda a, b: a & b, "difference": lambda a, b: a - b}


@pytest.mark.parametrize("op", ["union", "intersect", "difference"])
def test_table1_worked_examples(op):
    g = GOLD[op]
    X = rel_from_rows(g["types"], g["left"])
    Y = rel_from_rows(g["types"], g["right"])
    assert oracle.setop(X, Y, op).rows() == [tuple(r) for r in g["output"]]


def test_exhaustive_small_relations_vs_python_sets():
    """Every sorted bag of <= 3 tuples over {0,1,2} x {0,1} (duplicates included) on
    both sides, all three operators, against Python set algebra."""
    tuples = sorted(product([0, 1, 2], [0, 1]))
    rels = []
    for n in range(4):
        for rows in product(tuples, repeat=n):
            if list(rows) == sorted(rows):
                rels.append(list(rows))
    checked = 0
    for a in rels[::3]:
        for b in rels[::2]:
            X, Y = rel_from_rows(["i32", "u8"], a), rel_from_rows(["i32", "u8"], b)
            for op, f in PY.items():
                assert oracle.setop(X, Y, op).rows() == sorted(f(set(a), set(b))), (op, a, b)
                checked += 1
    assert checked > 3000


def random_sorted(rng, n, types, hi):
    cols = [rng.integers(-hi if t.startswith("i") else 0, hi, n).astype(oracle.NP[t]) for t in types]
    order = np.lexsort(cols[::-1])
    return oracle.Relation(types, [c[order] for c in cols])


@pytest.mark.parametrize("types", [["i32", "i32"], ["u32", "u8", "i64"], ["i64"], ["u64", "i32"]])
def test_large_random_vs_numpy_unique(types):
    rng = np.random.default_rng(7)
    X = random_sorted(rng, 40_000, types, 60)
    Y = random_sorted(rng, 30_000, types, 60)
    dt = np.dtype([(f"f{i}", oracle.NP[t]) for i, t in enumerate(types)])

    def rec(R):
        a = np.empty(R.n, dtype=dt)
        for i, c in enumerate(R.cols):
            a[f"f{i}"] = c
        return a
    ux, uy = np.unique(rec(X)), np.unique(rec(Y))
    ref = {"union": np.union1d(ux, uy), "intersect": np.intersect1d(ux, uy),
           "difference": np.setdiff1d(ux, uy)}
    for op, r in ref.items():
        got = oracle.setop(X, Y, op)
        assert got.n == len(r)
        for i, c in enumerate(got.cols):
            assert np.array_equal(c, r[f"f{i}"]), op


def test_set_algebra_identities():
    rng = np.random.default_rng(11)
    X = random_sorted(rng, 5000, ["i32", "u32"], 30)
    Y = random_sorted(rng, 4000, ["i32", "u32"], 30)
    E = random_sorted(rng, 0, ["i32", "u32"], 30)
    dX = oracle.setop(X, E, "union")                       # distinct(X)
    assert dX.rows() == sorted(set(X.rows()))
    assert oracle.setop(X, X, "difference").n == 0
    assert oracle.setop(X, X, "intersect").rows() == dX.rows()
    u, i = oracle.setop(X, Y, "union"), oracle.setop(X, Y, "intersect")
    dxy, dyx = oracle.setop(X, Y, "difference"), oracle.setop(Y, X, "difference")
    assert u.n == i.n + dxy.n + dyx.n                      # disjoint decomposition of the union
    assert sorted(dxy.rows() + i.rows()) == dX.rows()       # (X - Y) + (X & Y) = X
    assert oracle.setop(Y, X, "union").rows() == u.rows()  # commutative
    assert oracle.setop(Y, X, "intersect").rows() == i.rows()


def test_signed_order_and_errors():
    X = rel_from_rows(["i32"], [[-5], [-1], [3]])
    Y = rel_from_rows(["i32"], [[-2], [-1]])
    assert oracle.setop(X, Y, "union").rows() == [(-5,), (-2,), (-1,), (3,)]
    with pytest.raises(oracle.OracleError) as e:
        oracle.setop(rel_from_rows(["i32"], [[3], [1]]), Y, "union")
    assert e.value.code == "unsorted"
    with pytest.raises(oracle.OracleError) as e:
        oracle.setop(rel_from_rows(["u32"], [[1]]), Y, "union")
    assert e.value.code == "type"
