"""Thin ctypes binding of librw.so (include/rw.h).  Argument marshalling only:
every step of the hot path runs in the library's sm_100a kernels.  torch is used
for device memory and streams.  There is no CPU fallback — if librw.so is missing
or no B200 is visible, the calls raise.
"""
from __future__ import annotations

import ctypes
import os
from typing import List, Optional, Sequence, Tuple

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "librw.so")

TYPES = {"i32": 0, "u32": 1, "i64": 2, "u64": 3, "u8": 4}
TYPE_NAMES = {v: k for k, v in TYPES.items()}
WIDTH = {"i32": 4, "u32": 4, "i64": 8, "u64": 8, "u8": 1}
CMP = {"<": 0, "<=": 1, ">": 2, ">=": 3, "==": 4, "!=": 5}
SETOPS = {"union": 0, "intersect": 1, "difference": 2}
EXPR = {"col": 0, "const": 1, "add": 2, "sub": 3, "mul": 4, "divc": 5}
STATUS = {0: "RW_OK", -1: "RW_E_ARG", -2: "RW_E_TYPE", -3: "RW_E_UNSORTED", -4: "RW_E_OVERFLOW",
          -5: "RW_E_UNSUPPORTED", -6: "RW_E_CAPACITY", -7: "RW_E_OOM", -8: "RW_E_CUDA",
          -9: "RW_E_DOMAIN", -10: "RW_E_STATE"}


class RwError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status
        self.name = STATUS.get(status, str(status))


class rw_pred(ctypes.Structure):
    _fields_ = [("col", ctypes.c_int32), ("op", ctypes.c_int32), ("rhs_is_col", ctypes.c_int32),
                ("rhs_col", ctypes.c_int32), ("rhs_const", ctypes.c_int64)]


class rw_expr(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("type", ctypes.c_int32), ("a", ctypes.c_int32),
                ("b", ctypes.c_int32), ("k", ctypes.c_int64)]


class rw_agg(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("col", ctypes.c_int32)]


class rw_plan_opts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("cuda_stream", ctypes.c_void_p), ("fuse", ctypes.c_int32),
                ("zero_copy_project", ctypes.c_int32), ("stages", ctypes.c_int32),
                ("ctas_per_sm", ctypes.c_int32), ("strict_overflow", ctypes.c_int32),
                ("host_chunk_log2", ctypes.c_int32), ("reserved", ctypes.c_int32 * 8)]


class rw_relation_in(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("cols", ctypes.POINTER(ctypes.c_void_p))]


class rw_relation_out(ctypes.Structure):
    _fields_ = [("cols", ctypes.POINTER(ctypes.c_void_p)), ("capacity", ctypes.c_int64),
                ("n_dev", ctypes.c_void_p), ("n", ctypes.c_int64)]


EXPORTS = ["rw_plan_create", "rw_plan_destroy", "rw_plan_add_input", "rw_plan_add_select",
           "rw_plan_add_project", "rw_plan_add_join", "rw_plan_add_setop", "rw_plan_add_agg", "rw_plan_node_schema",
           "rw_plan_execute", "rw_plan_execute_multi", "rw_plan_execute_host", "rw_plan_explain", "rw_plan_last_launches",
           "rw_status_str", "rw_last_error", "rw_split_by_splitters", "rw_merge_runs",
           "rw_pack_tuples", "rw_merge_packed_runs",
           "rw_plan_agg_limbs", "rw_plan_agg_export", "rw_plan_agg_import"]

_lib = None


def lib():
    """Load librw.so (fails loudly when it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback exists)")
    L = ctypes.CDLL(LIB_PATH)
    P = ctypes.POINTER
    i32, i64, vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_void_p
    L.rw_plan_create.argtypes = [P(vp), P(rw_plan_opts)]
    L.rw_plan_destroy.argtypes = [vp]
    L.rw_plan_destroy.restype = None
    L.rw_plan_add_input.argtypes = [vp, i32, P(i32), i32, P(i64), P(i64), P(i32)]
    L.rw_plan_add_select.argtypes = [vp, i32, P(rw_pred), i32, P(i32)]
    L.rw_plan_add_project.argtypes = [vp, i32, P(rw_expr), i32, P(i32), i32, P(i32)]
    L.rw_plan_add_join.argtypes = [vp, i32, i32, i32, P(i32)]
    L.rw_plan_add_setop.argtypes = [vp, i32, i32, i32, P(i32)]
    L.rw_plan_add_agg.argtypes = [vp, i32, P(i32), P(i32), i32, P(rw_agg), i32, P(i32)]
    L.rw_plan_node_schema.argtypes = [vp, i32, P(i32), P(i32)]
    L.rw_plan_execute.argtypes = [vp, P(rw_relation_in), i32, i32, P(rw_relation_out)]
    L.rw_plan_execute_host.argtypes = [vp, P(rw_relation_in), i32, i32, P(rw_relation_out)]
    L.rw_plan_execute_multi.argtypes = [vp, P(rw_relation_in), i32, P(i32), i32, P(rw_relation_out)]
    L.rw_plan_explain.argtypes = [vp, i32, ctypes.c_char_p, ctypes.c_size_t]
    L.rw_plan_last_launches.argtypes = [vp]
    L.rw_plan_last_launches.restype = i64
    L.rw_status_str.argtypes = [i32]
    L.rw_status_str.restype = ctypes.c_char_p
    L.rw_last_error.restype = ctypes.c_char_p
    L.rw_split_by_splitters.argtypes = [vp, i64, i32, vp, i32, vp, vp]
    L.rw_merge_runs.argtypes = [P(vp), P(i32), i32, P(i64), i32, P(vp), vp]
    L.rw_pack_tuples.argtypes = [P(vp), P(i32), i32, i64, vp, vp]
    L.rw_merge_packed_runs.argtypes = [vp, P(i32), i32, P(i64), i32, P(vp), vp]
    L.rw_plan_agg_limbs.argtypes = [vp, i32, P(i64)]
    L.rw_plan_agg_export.argtypes = [vp, i32, P(vp), vp, i64, vp]
    L.rw_plan_agg_import.argtypes = [vp, i32, vp, P(rw_relation_out)]
    for f in ["rw_plan_create", "rw_plan_add_input", "rw_plan_add_select", "rw_plan_add_project",
              "rw_plan_add_join", "rw_plan_add_setop", "rw_plan_add_agg", "rw_plan_node_schema", "rw_plan_execute",
              "rw_plan_execute_host", "rw_plan_execute_multi", "rw_plan_explain", "rw_split_by_splitters", "rw_merge_runs",
              "rw_pack_tuples", "rw_merge_packed_runs", "rw_plan_agg_limbs", "rw_plan_agg_export", "rw_plan_agg_import"]:
        getattr(L, f).restype = i32
    _lib = L
    return L


def check(st: int):
    if st != 0:
        raise RwError(st, lib().rw_last_error().decode())


def _i32arr(v):
    return (ctypes.c_int32 * max(1, len(v)))(*v)


def make_preds(preds):
    arr = (rw_pred * max(1, len(preds)))()
    for i, (col, op, rhs) in enumerate(preds):
        arr[i].col, arr[i].op = col, CMP[op]
        if isinstance(rhs, tuple):
            arr[i].rhs_is_col, arr[i].rhs_col = 1, rhs[1]
        else:
            arr[i].rhs_const = int(rhs)
    return arr


def make_exprs(exprs):
    arr = (rw_expr * max(1, len(exprs)))()
    for i, e in enumerate(exprs):
        arr[i].op, arr[i].type = EXPR[e[0]], TYPES[e[-1]]
        if e[0] == "col":
            arr[i].a = e[1]
        elif e[0] == "const":
            arr[i].k = int(e[1])
        elif e[0] == "divc":
            arr[i].a, arr[i].k = e[1], int(e[2])
        else:
            arr[i].a, arr[i].b = e[1], e[2]
    return arr


def _ptr(t) -> int:
    return t if isinstance(t, int) else t.data_ptr()


class Plan:
    """rw_plan_* with the same names; expressions / predicates use the oracle's
    plain-data spelling (see oracle/__init__.py docstring)."""

    def __init__(self, device: int = 0, stream=None, fuse: bool = True, zero_copy_project: bool = False,
                 stages: int = 0, ctas_per_sm: int = 0, strict_overflow: bool = False, defer: int = 0,
                 dbg: int = 0, dbg_ts: int = 0, items: int = 0, variant: int = 0,
                 gring: int = 0, agg_mode: int = 0, host_chunk_log2: int = 0):
        import torch
        if stream is None:
            stream = torch.cuda.current_stream(device)
        self.stream = stream
        o = rw_plan_opts()
        o.device = device
        o.cuda_stream = ctypes.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))
        o.fuse = 1 if fuse else 0
        o.zero_copy_project = 1 if zero_copy_project else 0
        o.stages, o.ctas_per_sm = stages, ctas_per_sm
        o.strict_overflow = 1 if strict_overflow else 0
        o.host_chunk_log2 = host_chunk_log2  # execute_host: 2^this rows per streamed chunk (0 = 2^25)
        o.reserved[0] = defer              # scan kernel store delay in tiles (0 = auto)
        o.reserved[1] = dbg                # diagnostics only (1: no look-back, 2: stream only, 4: timestamps)
        o.reserved[2] = ctypes.c_int32(dbg_ts & 0xffffffff).value
        o.reserved[3] = ctypes.c_int32((dbg_ts >> 32) & 0xffffffff).value
        o.reserved[5] = items              # tuning: rows per thread of the scan tile (0 = auto)
        o.reserved[4] = variant            # tuning: 2 = 512x4, 3 = 512x8 compute threads x rows
        # kernel / fusion switches (diagnostics and A/B measurements): 2 = L2-ring scan kernel
        # with its ring in shared memory, 3 = L2-ring scan kernel for every compacting chain,
        # 5 = no JOIN -> JOIN fusion, 6 = cp.async join gathers, 7 = no SELECT / PROJECT
        # fusion upstream of a JOIN, 8 / 9 = emitting kernel with only its shared / only its
        # L2 ring, 10 = emitting kernel for every compacting chain
        o.reserved[6] = gring
        o.reserved[7] = agg_mode           # 1 = force the thread-private-partials aggregate terminal, 2 = no fused Q1 row path
        self.device = device
        h = ctypes.c_void_p()
        check(lib().rw_plan_create(ctypes.byref(h), ctypes.byref(o)))
        self.h = h
        self.inputs: List[List[str]] = []

    def close(self):
        if getattr(self, "h", None):
            lib().rw_plan_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- construction ---------------------------------------------------
    def add_input(self, types: Sequence[str], nkey_sorted: int = 0, lo=None, hi=None) -> int:
        t = _i32arr([TYPES[x] for x in types])
        lo_a = (ctypes.c_int64 * len(types))(*lo) if lo is not None else None
        hi_a = (ctypes.c_int64 * len(types))(*hi) if hi is not None else None
        node = ctypes.c_int32()
        check(lib().rw_plan_add_input(self.h, len(types), t, nkey_sorted, lo_a, hi_a, ctypes.byref(node)))
        self.inputs.append(list(types))
        return node.value

    def add_select(self, in_node: int, preds) -> int:
        node = ctypes.c_int32()
        check(lib().rw_plan_add_select(self.h, in_node, make_preds(preds), len(preds), ctypes.byref(node)))
        return node.value

    def add_project(self, in_node: int, exprs, roots) -> int:
        node = ctypes.c_int32()
        check(lib().rw_plan_add_project(self.h, in_node, make_exprs(exprs), len(exprs), _i32arr(roots),
                                        len(roots), ctypes.byref(node)))
        return node.value

    def add_join(self, left: int, right: int, nkey: int = 1) -> int:
        node = ctypes.c_int32()
        check(lib().rw_plan_add_join(self.h, left, right, nkey, ctypes.byref(node)))
        return node.value

    def add_setop(self, left: int, right: int, op: str) -> int:
        """op: "union" | "intersect" | "difference" (left minus right)."""
        n = ctypes.c_int32()
        check(lib().rw_plan_add_setop(self.h, left, right, SETOPS[op], ctypes.byref(n)))
        return n.value

    def add_agg(self, in_node: int, gcols, gdomain, aggs) -> int:
        a = (rw_agg * max(1, len(aggs)))()
        for i, x in enumerate(aggs):
            a[i].op = 0 if x[0] == "count" else 1
            a[i].col = x[1] if x[0] == "sum" else 0
        node = ctypes.c_int32()
        check(lib().rw_plan_add_agg(self.h, in_node, _i32arr(gcols), _i32arr(gdomain), len(gcols), a,
                                    len(aggs), ctypes.byref(node)))
        return node.value

    def node_schema(self, node: int) -> List[str]:
        n = ctypes.c_int32()
        t = (ctypes.c_int32 * 32)()
        check(lib().rw_plan_node_schema(self.h, node, ctypes.byref(n), t))
        return [TYPE_NAMES[t[i]] for i in range(n.value)]

    # -- execution ------------------------------------------------------
    @staticmethod
    def _inputs(inputs):
        keep, arr = [], (rw_relation_in * max(1, len(inputs)))()
        for i, (n, cols) in enumerate(inputs):
            c = (ctypes.c_void_p * max(1, len(cols)))(*[_ptr(x) for x in cols])
            keep.append(c)
            arr[i].n = int(n)
            arr[i].cols = ctypes.cast(c, ctypes.POINTER(ctypes.c_void_p))
        return arr, keep

    def execute(self, inputs, out_node: int, out_cols, capacity: int, n_dev=None) -> Optional[int]:
        """inputs: [(n, [device tensor or pointer per column])]; out_cols: device tensors /
        pointers with `capacity` rows.  Returns the row count (synchronising) or None when
        n_dev (a device int64 tensor / pointer) receives it asynchronously."""
        arr, keep = self._inputs(inputs)
        oc = (ctypes.c_void_p * max(1, len(out_cols)))(*[_ptr(x) for x in out_cols])
        out = rw_relation_out(ctypes.cast(oc, ctypes.POINTER(ctypes.c_void_p)), int(capacity),
                              ctypes.c_void_p(_ptr(n_dev)) if n_dev is not None else None, -1)
        check(lib().rw_plan_execute(self.h, arr, len(inputs), out_node, ctypes.byref(out)))
        return None if n_dev is not None else out.n

    def execute_multi(self, inputs, out_nodes, out_cols, capacities, n_devs=None):
        """Input-dependence fusion: out_cols[k] / capacities[k] (/ n_devs[k]) receive
        out_nodes[k].  Returns the row counts (synchronising) or None with n_devs."""
        arr, keep = self._inputs(inputs)
        k = len(out_nodes)
        outs = (rw_relation_out * k)()
        for i in range(k):
            oc = (ctypes.c_void_p * max(1, len(out_cols[i])))(*[_ptr(x) for x in out_cols[i]])
            keep.append(oc)
            outs[i].cols = ctypes.cast(oc, ctypes.POINTER(ctypes.c_void_p))
            outs[i].capacity = int(capacities[i])
            outs[i].n_dev = _ptr(n_devs[i]) if n_devs is not None else None
            outs[i].n = -1
        check(lib().rw_plan_execute_multi(self.h, arr, len(inputs), _i32arr(out_nodes), k, outs))
        return None if n_devs is not None else [outs[i].n for i in range(k)]

    def run_multi(self, inputs, out_nodes, capacity: Optional[int] = None):
        """Allocate torch outputs for every node, execute_multi, return [(tensors, n)]."""
        import torch
        if capacity is None:
            capacity = max([int(n) for n, _ in inputs] + [1])
        dt = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64,
              "u8": torch.uint8}
        cols = [[torch.empty(max(capacity, 1), dtype=dt[t], device=f"cuda:{self.device}")
                 for t in self.node_schema(nd)] for nd in out_nodes]
        ns = self.execute_multi(inputs, out_nodes, cols, [capacity] * len(out_nodes))
        return [([c[:n] for c in cs], n) for cs, n in zip(cols, ns)]

    def execute_host(self, inputs, out_node: int, out_cols, capacity: int) -> int:
        """Same with HOST buffers (numpy arrays / pinned torch tensors / pointers)."""
        def hp(x):
            if isinstance(x, int):
                return x
            if hasattr(x, "data_ptr"):
                return x.data_ptr()
            return x.ctypes.data
        arr, keep = self._inputs([(n, [hp(c) for c in cols]) for n, cols in inputs])
        oc = (ctypes.c_void_p * max(1, len(out_cols)))(*[hp(x) for x in out_cols])
        out = rw_relation_out(ctypes.cast(oc, ctypes.POINTER(ctypes.c_void_p)), int(capacity), None, -1)
        check(lib().rw_plan_execute_host(self.h, arr, len(inputs), out_node, ctypes.byref(out)))
        return out.n

    def explain(self, out_node: int) -> str:
        buf = ctypes.create_string_buffer(1 << 16)
        check(lib().rw_plan_explain(self.h, out_node, buf, len(buf)))
        return buf.value.decode()

    # -- aggregate combine across row shards -------------------------------
    def agg_limbs(self, node: int) -> int:
        n = ctypes.c_int64()
        check(lib().rw_plan_agg_limbs(self.h, node, ctypes.byref(n)))
        return n.value

    def agg_export(self, node: int, cols, n_dev=None, n_host: int = 0, limbs=None):
        """Local aggregate result -> dense int64 limbs (device tensor, returned)."""
        import torch
        if limbs is None:
            limbs = torch.empty(self.agg_limbs(node), dtype=torch.int64, device=f"cuda:{self.device}")
        c = (ctypes.c_void_p * len(cols))(*[_ptr(x) for x in cols])
        check(lib().rw_plan_agg_export(self.h, node, c, ctypes.c_void_p(_ptr(n_dev)) if n_dev is not None else None,
                                       int(n_host), ctypes.c_void_p(_ptr(limbs))))
        return limbs

    def agg_import(self, node: int, limbs, out_cols, capacity: int, n_dev=None):
        oc = (ctypes.c_void_p * max(1, len(out_cols)))(*[_ptr(x) for x in out_cols])
        out = rw_relation_out(ctypes.cast(oc, ctypes.POINTER(ctypes.c_void_p)), int(capacity),
                              ctypes.c_void_p(_ptr(n_dev)) if n_dev is not None else None, -1)
        check(lib().rw_plan_agg_import(self.h, node, ctypes.c_void_p(_ptr(limbs)), ctypes.byref(out)))
        return None if n_dev is not None else out.n

    def last_launches(self) -> int:
        return int(lib().rw_plan_last_launches(self.h))

    # -- convenience (allocation only) -----------------------------------
    def run(self, inputs, out_node: int, capacity: Optional[int] = None):
        """Allocate torch output columns, execute, return (list of tensors trimmed to n, n)."""
        import torch
        types = self.node_schema(out_node)
        if capacity is None:
            capacity = max([int(n) for n, _ in inputs] + [1])
        dt = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64,
              "u8": torch.uint8}
        outs = [torch.empty(max(capacity, 1), dtype=dt[t], device=f"cuda:{self.device}") for t in types]
        n = self.execute(inputs, out_node, outs, capacity)
        return [o[:n] for o in outs], n


def split_by_splitters(keys, n: int, key_type: str, splitters, nsplit: int, bounds, stream) -> None:
    check(lib().rw_split_by_splitters(ctypes.c_void_p(_ptr(keys)), n, TYPES[key_type],
                                      ctypes.c_void_p(_ptr(splitters)), nsplit, ctypes.c_void_p(_ptr(bounds)),
                                      ctypes.c_void_p(stream.cuda_stream)))


def merge_runs(cols, types, run_off, out_cols, stream) -> None:
    c = (ctypes.c_void_p * len(cols))(*[_ptr(x) for x in cols])
    t = _i32arr([TYPES[x] for x in types])
    ro = (ctypes.c_int64 * len(run_off))(*[int(x) for x in run_off])
    o = (ctypes.c_void_p * len(out_cols))(*[_ptr(x) for x in out_cols])
    check(lib().rw_merge_runs(c, t, len(cols), ro, len(run_off) - 1, o, ctypes.c_void_p(stream.cuda_stream)))


def pack_tuples(cols, types, n: int, packed, stream) -> None:
    c = (ctypes.c_void_p * len(cols))(*[_ptr(x) for x in cols])
    t = _i32arr([TYPES[x] for x in types])
    check(lib().rw_pack_tuples(c, t, len(cols), n, ctypes.c_void_p(_ptr(packed)), ctypes.c_void_p(stream.cuda_stream)))


def merge_packed_runs(packed, types, run_off, out_cols, stream) -> None:
    t = _i32arr([TYPES[x] for x in types])
    ro = (ctypes.c_int64 * len(run_off))(*[int(x) for x in run_off])
    o = (ctypes.c_void_p * len(out_cols))(*[_ptr(x) for x in out_cols])
    check(lib().rw_merge_packed_runs(ctypes.c_void_p(_ptr(packed)), t, len(types), ro, len(run_off) - 1, o,
                                     ctypes.c_void_p(stream.cuda_stream)))
