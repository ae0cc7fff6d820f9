"""Pins for oracle group-by aggregate (oracle.c or_agg; P:258-266 Q1, readings A10-A12)."""
import numpy as np
import pytest

import oracle
import rwgen
from tests import bruteforce as bf


def q1_sums(rel):
    """(rf, ls) -> [count, sum_qty, sum_price, sum_disc] as python ints via or_agg."""
    out = oracle.agg(rel, [5, 6], [3, 2], [("count",), ("sum", 1), ("sum", 2), ("sum", 3)])
    res = {}
    for i in range(out.n):
        g = (int(out.cols[0][i]), int(out.cols[1][i]))
        s = [int(out.cols[2][i])]
        for k in range(3):
            s.append(oracle.sum128(out.cols[3 + 2 * k][i:i + 1], out.cols[4 + 2 * k][i:i + 1])[0])
        res[g] = s
    return res


def lineitem_rel(n, cfg=0x84, start=0):
    li = rwgen.lineitem(cfg, start, n)
    names = ["shipdate", "qty", "price", "disc", "tax", "rf", "ls"]
    types = ["i32", "i64", "i64", "i64", "i64", "u8", "u8"]
    return oracle.Relation(types, [li[k].numpy() for k in names])


def test_brute_force_small():
    rng = np.random.default_rng(11)
    for _ in range(30):
        n = int(rng.integers(0, 40))
        g1 = rng.integers(0, 3, n)
        g2 = rng.integers(0, 2, n)
        v = rng.integers(-2**40, 2**40, n)
        rows = list(zip(g1.tolist(), g2.tolist(), v.tolist()))
        rel = oracle.Relation(["u8", "u32", "i64"], [g1, g2, v])
        out = oracle.agg(rel, [0, 1], [3, 2], [("count",), ("sum", 2)])
        got = [(a, b, c, s) for (a, b, c), s in zip(zip(out.cols[0].tolist(), out.cols[1].tolist(),
                                                          out.cols[2].tolist()),
                                                      oracle.sum128(out.cols[3], out.cols[4]))]
        assert got == bf.group_sum(rows, [0, 1], [3, 2], [("count",), ("sum", 2)])


def test_count_and_sum_invariants_and_additivity():
    rel = lineitem_rel(30000)
    res = q1_sums(rel)
    assert sum(v[0] for v in res.values()) == rel.n
    assert sum(v[1] for v in res.values()) == int(rel.cols[1].sum())      # numpy int64 sum
    assert sum(v[2] for v in res.values()) == int(rel.cols[2].sum())
    # additivity: Q1(R1 + R2) == Q1(R1) + Q1(R2)
    a = lineitem_rel(12000, start=0)
    b = lineitem_rel(18000, start=12000)
    ra, rb = q1_sums(a), q1_sums(b)
    for g, v in res.items():
        va = ra.get(g, [0] * 4)
        vb = rb.get(g, [0] * 4)
        assert v == [x + y for x, y in zip(va, vb)]
    # only groups that occur, ascending (rf, ls)  — reading A12
    assert list(res) == sorted(res)


def test_128bit_exact_beyond_int64():
    v = np.full(8, 2**62 + 12345, np.int64)
    g = np.zeros(8, np.uint8)
    out = oracle.agg(oracle.Relation(["u8", "i64"], [g, v]), [0], [1], [("sum", 1)])
    assert oracle.sum128(out.cols[1], out.cols[2]) == [8 * (2**62 + 12345)]
    neg = np.full(8, -2**63, np.int64)
    out = oracle.agg(oracle.Relation(["u8", "i64"], [g, neg]), [0], [1], [("sum", 1)])
    assert oracle.sum128(out.cols[1], out.cols[2]) == [-8 * 2**63]
    u = np.full(5, 2**64 - 1, np.uint64)
    out = oracle.agg(oracle.Relation(["u8", "u64"], [g[:5], u]), [0], [1], [("sum", 1)])
    assert oracle.sum128(out.cols[1], out.cols[2]) == [5 * (2**64 - 1)]


def test_empty_and_no_groups_and_domain_error():
    e = oracle.Relation(["u8", "i64"], [np.zeros(0, np.uint8), np.zeros(0, np.int64)])
    assert oracle.agg(e, [0], [4], [("count",)]).n == 0
    r = oracle.Relation(["u8", "i64"], [np.array([0, 0, 1], np.uint8), np.array([1, 2, 3], np.int64)])
    out = oracle.agg(r, [], [], [("count",), ("sum", 1)])     # global aggregate: one group
    assert out.rows() == [(3, 6, 0)]
    bad = oracle.Relation(["u8"], [np.array([0, 5], np.uint8)])
    with pytest.raises(oracle.OracleError) as ei:
        oracle.agg(bad, [0], [3], [("count",)])
    assert ei.value.code == "domain"
