"""Plan specs and seeded inputs for the BASELINE.json configurations (C1..C5).

Plain data only: a spec names the operators and their constants (SURVEY.md §8(d)
table, readings A13-A17).  It is consumed by the oracle (oracle.evaluate) and by
tests/planspec.py / bench.py for the CUDA path.  Inputs come from rwgen.
"""
from __future__ import annotations

from typing import Dict, List

import rwgen

C1_ROWS = 1 << 20
C2_ROWS = 1 << 29
C3_ROWS = 1 << 26
C4_ROWS = 600_000_000
C5_ROWS = 1 << 30


def thr_u32(s: float) -> int:
    """u32 threshold T with P(x < T) = s for uniform x (reading A13)."""
    return int(s * (1 << 32))


def thr_i32(s: float) -> int:
    return -(1 << 31) + int(s * (1 << 32))


# ---- C1: two back-to-back SELECTs over (u32 key, u32 val) ---------------------
def c1_spec(s1: float = 0.5, s2: float = 0.5) -> Dict:
    return {"inputs": {"R": {"types": ["u32", "u32"], "nkey_sorted": 0}},
            "nodes": [{"id": "s1", "op": "select", "in": "R", "preds": [(0, "<", thr_u32(s1))]},
                      {"id": "s2", "op": "select", "in": "s1", "preds": [(1, "<", thr_u32(s2))]}],
            "out": "s2"}


def c1_inputs(n: int, start: int = 0, device="cpu", cfg: int = 1) -> Dict[str, List]:
    r = rwgen.uniform_u32_relation(cfg, 0, 2, start, n, device)
    return {"R": [r["c0"], r["c1"]]}


# ---- C2: SELECT -> PROJECT -> SELECT over 4 x i32 ------------------------------
def c2_spec(s1: float = 0.5, s2: float = 0.5) -> Dict:
    return {"inputs": {"R": {"types": ["i32"] * 4, "nkey_sorted": 0}},
            "nodes": [{"id": "s1", "op": "select", "in": "R", "preds": [(1, "<", thr_i32(s1))]},
                      {"id": "p", "op": "project", "in": "s1",
                       "exprs": [("col", 0, "i32"), ("col", 2, "i32"), ("col", 3, "i32")], "roots": [0, 1, 2]},
                      {"id": "s2", "op": "select", "in": "p", "preds": [(2, "<", thr_i32(s2))]}],
            "out": "s2"}


def c2_inputs(n: int, start: int = 0, device="cpu", cfg: int = 2) -> Dict[str, List]:
    r = rwgen.uniform_u32_relation(cfg, 0, 4, start, n, device)
    return {"R": [r[f"c{c}"] for c in range(4)]}


# ---- pattern (d): input dependence (§4.4, Fig. 14(d)) ------------
# k SELECTs filter the same 16-byte tuples; branch b keeps the rows with
# c_b < threshold (selectivity s each, reading A13) and all four columns.
def cd_spec(s: float = 0.25, k: int = 2) -> Dict:
    nodes = [{"id": f"d{b}", "op": "select", "in": "R", "preds": [(b, "<", thr_i32(s))]} for b in range(k)]
    return {"inputs": {"R": {"types": ["i32"] * 4, "nkey_sorted": 0}}, "nodes": nodes,
            "outs": [f"d{b}" for b in range(k)], "out": "d0"}


def cd_inputs(n: int, start: int = 0, device="cpu", cfg: int = 6) -> Dict[str, List]:
    r = rwgen.uniform_u32_relation(cfg, 0, 4, start, n, device)
    return {"R": [r[f"c{c}"] for c in range(4)]}


# ---- set operators (Table 1) --------------------------
# x, y: n tuples (u32 key uniform in [0, n), u32 val in [0, 4)), each sorted on both
# columns; about 22 % of y's distinct tuples also occur in x.
def cs_spec(op: str = "union") -> Dict:
    return {"inputs": {"X": {"types": ["u32", "u32"], "nkey_sorted": 2},
                       "Y": {"types": ["u32", "u32"], "nkey_sorted": 2}},
            "nodes": [{"id": "s", "op": op, "left": "X", "right": "Y"}], "out": "s"}


def cs_inputs(n: int, device="cpu", cfg: int = 7, nval: int = 4, key_space: int = None,
              start: int = 0) -> Dict[str, List]:
    """Rows [start, start + n) of x and y (each returned sorted on both columns)."""
    ks = key_space or max(n, 1)
    X = rwgen.setop_relation(cfg, 0, n, ks, nval, device, start)
    Y = rwgen.setop_relation(cfg, 1, n, ks, nval, device, start)
    return {"X": [X["key"], X["val"]], "Y": [Y["key"], Y["val"]]}


# ---- C3: JOIN (Zipf 0.5) -> SELECT -> PROJECT ---------------------------------
def c3_spec() -> Dict:
    return {"inputs": {"L": {"types": ["u32", "u32"], "nkey_sorted": 1},
                       "R": {"types": ["u32", "u32"], "nkey_sorted": 1}},
            "nodes": [{"id": "j", "op": "join", "left": "L", "right": "R", "nkey": 1},
                      {"id": "s", "op": "select", "in": "j", "preds": [(1, "<", ("col", 2))]},
                      {"id": "p", "op": "project", "in": "s",
                       "exprs": [("col", 0, "u32"), ("col", 2, "u32")], "roots": [0, 1]}],
            "out": "p"}


def cc_spec() -> Dict:
    """Pattern (c) (Fig. 14(c), Fig. 13): SELECTs on the join key of both C3
    inputs, then the C3 join -> SELECT -> PROJECT.  Key ranges keep about half of L's
    and three quarters of R's keys (thresholds on the scattered key values)."""
    spec = c3_spec()
    spec["nodes"] = [{"id": "fl", "op": "select", "in": "L", "preds": [(0, "<", thr_u32(0.5))]},
                     {"id": "fr", "op": "select", "in": "R", "preds": [(0, ">=", thr_u32(0.25))]},
                     {"id": "j", "op": "join", "left": "fl", "right": "fr", "nkey": 1}] + spec["nodes"][1:]
    return spec


def c3_inputs(n: int, K: int = None, device="cpu", cfg: int = 3, cdf=None) -> Dict[str, List]:
    K = K or max(n, 1)
    if cdf is None and n > 0:
        cdf = rwgen.zipf_cdf(K, 0.5, device)
    L = rwgen.zipf_join_relation(cfg, 0, n, K, device, cdf)
    R = rwgen.zipf_join_relation(cfg, 1, n, K, device, cdf)
    return {"L": [L["key"], L["val"]], "R": [R["key"], R["val"]]}


# ---- C4: TPC-H Q1-shaped select / arithmetic / group-by ------------------------
Q1_COLS = ["shipdate", "qty", "price", "disc", "tax", "rf", "ls"]
Q1_TYPES = ["i32", "i64", "i64", "i64", "i64", "u8", "u8"]
# caller-declared value bounds of the generated lineitem (rwgen.lineitem)
Q1_LO = [rwgen.D_1992_01_01 + 1, 100, 0, 0, 0, 0, 0]
Q1_HI = [rwgen.D_1998_08_02 + 121, 5000, 10_495_000, 10, 8, 2, 1]


def c4_spec() -> Dict:
    exprs = [("col", 5, "u8"), ("col", 6, "u8"), ("col", 1, "i64"), ("col", 2, "i64"), ("col", 3, "i64"),
             ("col", 4, "i64"), ("const", 100, "i64"),
             ("sub", 6, 4, "i64"),          # 7: 100 - disc          (1 - discount, scale 2)
             ("mul", 3, 7, "i64"),          # 8: disc_price          (scale 4)
             ("add", 6, 5, "i64"),          # 9: 100 + tax           (1 + tax, scale 2)
             ("mul", 8, 9, "i64")]          # 10: charge             (scale 6)
    return {"inputs": {"lineitem": {"types": Q1_TYPES, "nkey_sorted": 0, "lo": Q1_LO, "hi": Q1_HI}},
            "nodes": [{"id": "s", "op": "select", "in": "lineitem", "preds": [(0, "<=", rwgen.D_1998_09_02)]},
                      {"id": "p", "op": "project", "in": "s", "exprs": exprs, "roots": [0, 1, 2, 3, 8, 10, 4]},
                      {"id": "g", "op": "agg", "in": "p", "gcols": [0, 1], "gdomain": [3, 2],
                       "aggs": [("count",), ("sum", 2), ("sum", 3), ("sum", 4), ("sum", 5), ("sum", 6)]}],
            "out": "g"}


def c4_inputs(n: int, start: int = 0, device="cpu", cfg: int = 4) -> Dict[str, List]:
    li = rwgen.lineitem(cfg, start, n, device=device)
    return {"lineitem": [li[c] for c in Q1_COLS]}


# ---- C5: JOIN -> JOIN -> SELECT over three relations --------------------------
def c5_spec() -> Dict:
    return {"inputs": {"R": {"types": ["u32", "u32"], "nkey_sorted": 1},
                       "S": {"types": ["u32", "u32"], "nkey_sorted": 1},
                       "T": {"types": ["u32", "u32"], "nkey_sorted": 1}},
            "nodes": [{"id": "rs", "op": "join", "left": "R", "right": "S", "nkey": 1},
                      {"id": "rst", "op": "join", "left": "rs", "right": "T", "nkey": 1},
                      {"id": "s", "op": "select", "in": "rst", "preds": [(1, "<", ("col", 3))]}],
            "out": "s"}


def c5_inputs(n: int, key_space: int = None, start: int = 0, device="cpu", cfg: int = 5) -> Dict[str, List]:
    key_space = key_space or max(n, 1)
    out = {}
    for rel, name in enumerate("RST"):
        r = rwgen.uniform_join_relation(cfg, rel, start, n, key_space, device)
        out[name] = [r["key"], r["val"]]
    return out


def input_bytes(spec: Dict, n_rows: Dict[str, int]) -> int:
    w = {"i32": 4, "u32": 4, "i64": 8, "u64": 8, "u8": 1}
    return sum(n_rows[k] * sum(w[t] for t in v["types"]) for k, v in spec["inputs"].items())
