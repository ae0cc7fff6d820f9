"""Pins for oracle PROJECT / arithmetic (oracle.c or_project)."""
import json
import os

import numpy as np
import pytest

import oracle
from tests.test_oracle_select import rel_from_rows

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table1.json")))


def test_table1_project_worked_example():
    g = GOLD["project"]
    r = rel_from_rows(g["types"], g["input"])
    exprs = [("col", c, g["types"][c]) for c in g["keep"]]
    out = oracle.project(r, exprs, list(range(len(exprs))))
    assert out.rows() == [tuple(x) for x in g["output"]]
    assert out.types == [g["types"][c] for c in g["keep"]]


@pytest.mark.parametrize("t,npt", [("i32", np.int32), ("u32", np.uint32), ("i64", np.int64), ("u64", np.uint64)])
def test_add_sub_mul_wrap_like_numpy(t, npt):
    # numpy fixed-width array arithmetic wraps mod 2^w: an independent implementation
    rng = np.random.default_rng(1)
    info = np.iinfo(npt)
    a = rng.integers(info.min, info.max, size=5000, dtype=npt, endpoint=True)
    b = rng.integers(info.min, info.max, size=5000, dtype=npt, endpoint=True)
    a[:4] = [info.min, info.max, 0, info.max]
    b[:4] = [info.min, info.max, info.min, 1]
    r = oracle.Relation([t, t], [a, b])
    ex = [("col", 0, t), ("col", 1, t), ("add", 0, 1, t), ("sub", 0, 1, t), ("mul", 0, 1, t)]
    out = oracle.project(r, ex, [2, 3, 4])
    with np.errstate(over="ignore"):
        assert np.array_equal(out.cols[0], a + b)
        assert np.array_equal(out.cols[1], a - b)
        assert np.array_equal(out.cols[2], a * b)


def test_divc_truncates_toward_zero():
    rng = np.random.default_rng(2)
    a = rng.integers(-2**31, 2**31, size=4000, dtype=np.int64).astype(np.int32)
    r = oracle.Relation(["i32"], [a])
    for k in (7, -7, 1, -1, 100):
        out = oracle.project(r, [("col", 0, "i32"), ("divc", 0, k, "i32")], [1])
        # np.fix on float64 is exact here (|a| < 2^53): library truncation toward zero
        expect = np.fix(a.astype(np.float64) / k)
        expect = np.where(expect == 2**31, -2**31, expect).astype(np.int64)   # MIN / -1 wraps
        assert np.array_equal(out.cols[0].astype(np.int64), expect)
    # i64: characterise truncated division by q*k + r == a, |r| < |k|, sign(r) in {0, sign(a)}
    a64 = rng.integers(-2**62, 2**62, size=2000, dtype=np.int64)
    r64 = oracle.Relation(["i64"], [a64])
    for k in (3, -1000003):
        q = oracle.project(r64, [("col", 0, "i64"), ("divc", 0, k, "i64")], [1]).cols[0]
        for x, y in zip(a64.tolist(), q.tolist()):
            rem = x - y * k
            assert abs(rem) < abs(k) and (rem == 0 or (rem > 0) == (x > 0))
    mn = oracle.Relation(["i64"], [np.array([-2**63], np.int64)])
    assert oracle.project(mn, [("col", 0, "i64"), ("divc", 0, -1, "i64")], [1]).rows() == [(-2**63,)]
    with pytest.raises(oracle.OracleError):
        oracle.project(mn, [("col", 0, "i64"), ("divc", 0, 0, "i64")], [1])


def test_type_conversion_of_column_refs():
    r = oracle.Relation(["i32", "u32"], [np.array([-1], np.int32), np.array([0xFFFFFFFF], np.uint32)])
    ex = [("col", 0, "u32"), ("col", 0, "i64"), ("col", 1, "i64"), ("col", 1, "i32")]
    assert oracle.project(r, ex, [0, 1, 2, 3]).rows() == [(0xFFFFFFFF, -1, 0xFFFFFFFF, -1)]


def test_q1_arithmetic_closed_forms():
    # pattern (e) P:223 price*(1-discount)*(1+tax) in fixed point (readings A8, A9):
    # disc = tax = 0  =>  charge = price * 100 * 100
    price = np.array([1, 99, 10495000, 123456], np.int64)
    zero = np.zeros(4, np.int64)
    r = oracle.Relation(["i64", "i64", "i64"], [price, zero, zero])
    ex = [("col", 0, "i64"), ("col", 1, "i64"), ("col", 2, "i64"), ("const", 100, "i64"),
          ("sub", 3, 1, "i64"), ("mul", 0, 4, "i64"), ("add", 3, 2, "i64"), ("mul", 5, 6, "i64")]
    out = oracle.project(r, ex, [5, 7])
    assert out.cols[0].tolist() == (price * 100).tolist()
    assert out.cols[1].tolist() == (price * 10000).tolist()


def test_identity_and_composition():
    rng = np.random.default_rng(3)
    cols = [rng.integers(0, 2**32, size=1000, dtype=np.uint64).astype(np.uint32) for _ in range(4)]
    r = oracle.Relation(["u32"] * 4, cols)
    ident = oracle.project(r, [("col", c, "u32") for c in range(4)], [0, 1, 2, 3])
    assert ident.rows() == r.rows()
    a = [3, 0, 2]                      # pi_a after pi_b == pi_{b o a}
    b = [1, 3, 0, 2]
    pb = oracle.project(r, [("col", c, "u32") for c in b], list(range(4)))
    pab = oracle.project(pb, [("col", c, "u32") for c in a], list(range(3)))
    direct = oracle.project(r, [("col", b[c], "u32") for c in a], list(range(3)))
    assert pab.rows() == direct.rows()
