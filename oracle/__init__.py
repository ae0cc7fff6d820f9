"""CPU oracle for the fused relational-algebra hot path — TEST INFRASTRUCTURE.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s cpu_baseline /
`--impl reference` legs may import this package.  The product path
(`paper_conf_micro_wudcy12_b200`) never imports it and shares no code with it.

`oracle.c` (same directory) is the evaluator: one operator at a time, every
intermediate materialised, single thread.  This module only marshals numpy
columns through ctypes and walks a plan spec in order (SURVEY.md §8(c) c2,
"a fused chain equals the composition of these, evaluated one operator at a
time with every intermediate materialized").

Parity pins: tests/test_oracle_select.py, test_oracle_project.py,
test_oracle_join.py, test_oracle_agg.py (Table 1 worked examples, brute force
on tiny inputs, cardinality invariants, closed forms).  Parity unpinned: none of
the functions here; see DESIGN.md §Oracle.

Plan spec (plain data, also consumed by tests/planspec.py for the CUDA side):
    {"inputs": {name: {"types": [...], "nkey_sorted": k}},
     "nodes": [{"id": .., "op": "select", "in": .., "preds": [(col, op, rhs)]},
               {"id": .., "op": "project", "in": .., "exprs": [...], "roots": [...]},
               {"id": .., "op": "join", "left": .., "right": .., "nkey": k},
               {"id": .., "op": "union" | "intersect" | "difference", "left": .., "right": ..},
               {"id": .., "op": "agg", "in": .., "gcols": [..], "gdomain": [..],
                "aggs": [("count",) | ("sum", col)]}],
     "out": id}
    rhs = int constant | ("col", j);  op in {"<","<=",">",">=","==","!="}
    exprs: ("col", c, type) | ("const", k, type) | (op, a, b, type) for op in
           add/sub/mul | ("divc", a, k, type); children index earlier exprs.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import time
from typing import Dict, List, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

MAXCOLS = 32
TYPES = {"i32": 0, "u32": 1, "i64": 2, "u64": 3, "u8": 4}
NP = {"i32": np.int32, "u32": np.uint32, "i64": np.int64, "u64": np.uint64, "u8": np.uint8}
TYPE_NAMES = {v: k for k, v in TYPES.items()}
CMP = {"<": 0, "<=": 1, ">": 2, ">=": 3, "==": 4, "!=": 5}
EXPR = {"col": 0, "const": 1, "add": 2, "sub": 3, "mul": 4, "divc": 5}
ERRORS = {-1: "arg", -2: "type", -3: "unsorted", -4: "domain", -5: "oom"}


class OracleError(RuntimeError):
    def __init__(self, rc):
        super().__init__(f"oracle error {rc} ({ERRORS.get(rc, '?')})")
        self.code = ERRORS.get(rc, str(rc))


class _Rel(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("ncols", ctypes.c_int32),
                ("types", ctypes.c_int32 * MAXCOLS), ("cols", ctypes.c_void_p * MAXCOLS)]


class _Pred(ctypes.Structure):
    _fields_ = [("col", ctypes.c_int32), ("op", ctypes.c_int32), ("rhs_is_col", ctypes.c_int32),
                ("rhs_col", ctypes.c_int32), ("rhs_const", ctypes.c_int64)]


class _Expr(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("type", ctypes.c_int32), ("a", ctypes.c_int32),
                ("b", ctypes.c_int32), ("k", ctypes.c_int64)]


class _Agg(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("col", ctypes.c_int32)]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so with plain gcc -O2 (no vectorisation flags)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-Wall",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P = ctypes.POINTER
        _lib.or_select.argtypes = [P(_Rel), ctypes.c_int32, P(_Pred), P(_Rel)]
        _lib.or_project.argtypes = [P(_Rel), ctypes.c_int32, P(_Expr), ctypes.c_int32,
                                    P(ctypes.c_int32), P(_Rel)]
        _lib.or_join.argtypes = [P(_Rel), P(_Rel), ctypes.c_int32, P(_Rel)]
        _lib.or_setop.argtypes = [P(_Rel), P(_Rel), ctypes.c_int32, P(_Rel)]
        _lib.or_agg.argtypes = [P(_Rel), ctypes.c_int32, P(ctypes.c_int32), P(ctypes.c_int32),
                                ctypes.c_int32, P(_Agg), P(_Rel)]
        _lib.or_free.argtypes = [P(_Rel)]
    return _lib


class Relation:
    """Host relation: list of typed numpy columns (SoA)."""

    def __init__(self, types: Sequence[str], cols: Sequence[np.ndarray]):
        assert len(types) == len(cols)
        self.types = list(types)
        self.cols = [np.ascontiguousarray(np.asarray(c).astype(NP[t], copy=False))
                     for t, c in zip(types, cols)]
        n = {len(c) for c in self.cols}
        assert len(n) <= 1, "ragged relation"
        self.n = n.pop() if n else 0

    def rows(self):
        return list(zip(*[c.tolist() for c in self.cols])) if self.cols else []

    def _c(self):
        r = _Rel()
        r.n = self.n
        r.ncols = len(self.cols)
        for i, (t, c) in enumerate(zip(self.types, self.cols)):
            r.types[i] = TYPES[t]
            r.cols[i] = c.ctypes.data
        return r


def _take(r: _Rel) -> Relation:
    types, cols = [], []
    for i in range(r.ncols):
        t = TYPE_NAMES[r.types[i]]
        a = np.empty(r.n, dtype=NP[t])
        if r.n:
            ctypes.memmove(a.ctypes.data, r.cols[i], r.n * a.itemsize)
        types.append(t)
        cols.append(a)
    lib().or_free(ctypes.byref(r))
    return Relation(types, cols)


def _check(rc):
    if rc != 0:
        raise OracleError(rc)


def select(rel: Relation, preds) -> Relation:
    arr = (_Pred * max(1, len(preds)))()
    for i, (col, op, rhs) in enumerate(preds):
        arr[i].col = col
        arr[i].op = CMP[op]
        if isinstance(rhs, tuple):
            arr[i].rhs_is_col, arr[i].rhs_col = 1, rhs[1]
        else:
            arr[i].rhs_const = int(rhs)
    out = _Rel()
    _check(lib().or_select(ctypes.byref(rel._c()), len(preds), arr, ctypes.byref(out)))
    return _take(out)


def _exprs(exprs):
    arr = (_Expr * max(1, len(exprs)))()
    for i, e in enumerate(exprs):
        arr[i].op = EXPR[e[0]]
        arr[i].type = TYPES[e[-1]]
        if e[0] == "col":
            arr[i].a = e[1]
        elif e[0] == "const":
            arr[i].k = int(e[1])
        elif e[0] == "divc":
            arr[i].a, arr[i].k = e[1], int(e[2])
        else:
            arr[i].a, arr[i].b = e[1], e[2]
    return arr


def project(rel: Relation, exprs, roots) -> Relation:
    roots_a = (ctypes.c_int32 * max(1, len(roots)))(*roots)
    out = _Rel()
    _check(lib().or_project(ctypes.byref(rel._c()), len(exprs), _exprs(exprs), len(roots),
                            roots_a, ctypes.byref(out)))
    return _take(out)


SETOPS = {"union": 0, "intersect": 1, "difference": 2}


def setop(X: Relation, Y: Relation, op: str) -> Relation:
    """SET UNION / INTERSECTION / DIFFERENCE (Table 1, reading A24): distinct
    whole tuples, both inputs sorted on every attribute, result ascending."""
    out = _Rel()
    _check(lib().or_setop(ctypes.byref(X._c()), ctypes.byref(Y._c()), SETOPS[op], ctypes.byref(out)))
    return _take(out)


def join(L: Relation, R: Relation, nkey: int = 1) -> Relation:
    out = _Rel()
    _check(lib().or_join(ctypes.byref(L._c()), ctypes.byref(R._c()), nkey, ctypes.byref(out)))
    return _take(out)


def agg(rel: Relation, gcols, gdomain, aggs) -> Relation:
    g = (ctypes.c_int32 * max(1, len(gcols)))(*gcols)
    d = (ctypes.c_int32 * max(1, len(gdomain)))(*gdomain)
    a = (_Agg * max(1, len(aggs)))()
    for i, x in enumerate(aggs):
        a[i].op = 0 if x[0] == "count" else 1
        a[i].col = x[1] if x[0] == "sum" else 0
    out = _Rel()
    _check(lib().or_agg(ctypes.byref(rel._c()), len(gcols), g, d, len(aggs), a, ctypes.byref(out)))
    return _take(out)


def evaluate(spec: Dict, inputs: Dict[str, Relation], keep_all: bool = False):
    """Evaluate a plan spec one operator at a time, materialising each node."""
    env: Dict[str, Relation] = dict(inputs)
    for nd in spec["nodes"]:
        op = nd["op"]
        if op == "select":
            env[nd["id"]] = select(env[nd["in"]], nd["preds"])
        elif op == "project":
            env[nd["id"]] = project(env[nd["in"]], nd["exprs"], nd["roots"])
        elif op in SETOPS:
            env[nd["id"]] = setop(env[nd["left"]], env[nd["right"]], op)
        elif op == "join":
            env[nd["id"]] = join(env[nd["left"]], env[nd["right"]], nd.get("nkey", 1))
        elif op == "agg":
            env[nd["id"]] = agg(env[nd["in"]], nd["gcols"], nd["gdomain"], nd["aggs"])
        else:
            raise ValueError(op)
    return env if keep_all else env[spec["out"]]


def timed_evaluate(spec: Dict, inputs: Dict[str, Relation]):
    """(result, seconds) — wall time of the evaluation only (inputs already on host)."""
    t0 = time.perf_counter()
    r = evaluate(spec, inputs)
    return r, time.perf_counter() - t0


def sum128(lo: np.ndarray, hi: np.ndarray) -> List[int]:
    """Recombine (lo u64, hi i64) aggregate columns into python ints."""
    return [int(h) * (1 << 64) + int(l) for l, h in zip(lo.tolist(), hi.tolist())]
