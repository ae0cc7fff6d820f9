"""Pins for oracle JOIN (oracle.c or_join; Table 1, reading A1)."""
import json
import os
from itertools import product

import numpy as np
import pytest

import oracle
import rwgen
from tests import bruteforce as bf
from tests.test_oracle_select import rel_from_rows

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table1.json")))


def test_table1_join_corrected_example():
    g = GOLD["join"]
    L = rel_from_rows(g["types"], g["left"])
    R = rel_from_rows(g["types"], g["right"])
    assert oracle.join(L, R).rows() == [tuple(x) for x in g["output"]]


def test_exhaustive_small_sorted_relations_vs_nested_loop():
    n_checked = 0
    keys = [0, 1, 2]
    tuples = sorted(product(keys, [0, 1]))
    rels = []
    for n in range(4):
        for rows in product(tuples, repeat=n):
            rows = sorted(rows)
            if rows not in rels:
                rels.append(rows)
    for Lrows in rels:
        L = rel_from_rows(["u32", "u32"], Lrows)
        for Rrows in rels[::2]:
            R = rel_from_rows(["u32", "u32"], Rrows)
            assert oracle.join(L, R).rows() == bf.nested_loop_join(Lrows, Rrows)
            n_checked += 1
    assert n_checked > 1000


def test_two_key_columns_vs_nested_loop():
    rng = np.random.default_rng(5)
    for _ in range(50):
        Lrows = sorted(tuple(int(x) for x in rng.integers(0, 3, 3)) for _ in range(rng.integers(0, 8)))
        Rrows = sorted(tuple(int(x) for x in rng.integers(0, 3, 3)) for _ in range(rng.integers(0, 8)))
        L = rel_from_rows(["i32"] * 3, Lrows)
        R = rel_from_rows(["i32"] * 3, Rrows)
        assert oracle.join(L, R, 2).rows() == bf.nested_loop_join(Lrows, Rrows, 2)


def test_join_size_is_sum_of_multiplicity_products():
    # |R join S| = sum_k m_R(k) m_S(k), computed with numpy.unique (library routine)
    n, K = 50000, 50000
    L = rwgen.zipf_join_relation(0x83, 0, n, K)
    R = rwgen.zipf_join_relation(0x83, 1, n, K)
    lk, rk = L["key"].numpy().view(np.uint32), R["key"].numpy().view(np.uint32)
    out = oracle.join(oracle.Relation(["u32", "u32"], [lk, L["val"].numpy().view(np.uint32)]),
                      oracle.Relation(["u32", "u32"], [rk, R["val"].numpy().view(np.uint32)]))
    ku, cu = np.unique(lk, return_counts=True)
    kv, cv = np.unique(rk, return_counts=True)
    common, il, ir = np.intersect1d(ku, kv, return_indices=True)
    assert out.n == int((cu[il].astype(np.int64) * cv[ir]).sum())
    # output is sorted by key and every output key occurs on both sides
    assert np.all(np.diff(out.cols[0].astype(np.int64)) >= 0)
    assert set(np.unique(out.cols[0]).tolist()) == set(common.tolist())


def test_unique_keys_full_match_is_column_glue():
    # P:266 "joining several columns together into a larger table"
    n = 1000
    k = np.arange(n, dtype=np.uint32) * 3
    a = np.arange(n, dtype=np.uint32) ^ 0x55
    b = np.arange(n, dtype=np.uint32) * 7
    out = oracle.join(oracle.Relation(["u32", "u32"], [k, a]), oracle.Relation(["u32", "u32"], [k, b]))
    assert out.n == n
    assert np.array_equal(out.cols[0], k) and np.array_equal(out.cols[1], a) and np.array_equal(out.cols[2], b)


def test_empty_side_and_errors():
    e = oracle.Relation(["u32", "u32"], [np.zeros(0, np.uint32)] * 2)
    x = oracle.Relation(["u32", "u32"], [np.array([1, 2], np.uint32)] * 2)
    assert oracle.join(e, x).n == 0 and oracle.join(x, e).n == 0
    uns = oracle.Relation(["u32", "u32"], [np.array([2, 1], np.uint32)] * 2)
    with pytest.raises(oracle.OracleError) as ei:
        oracle.join(uns, x)
    assert ei.value.code == "unsorted"
    y = oracle.Relation(["i32", "u32"], [np.array([1], np.int32), np.array([1], np.uint32)])
    with pytest.raises(oracle.OracleError) as ei:
        oracle.join(x, y)
    assert ei.value.code == "type"


def test_join_associative_up_to_column_order():
    rng = np.random.default_rng(9)
    def rel(n):
        k = np.sort(rng.integers(0, 20, n).astype(np.uint32))
        return oracle.Relation(["u32", "u32"], [k, rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)])
    R, S, T = rel(60), rel(50), rel(40)
    left = oracle.join(oracle.join(R, S), T)        # (k, r, s, t)
    right = oracle.join(R, oracle.join(S, T))       # (k, r, s, t)
    assert sorted(left.rows()) == sorted(right.rows())
