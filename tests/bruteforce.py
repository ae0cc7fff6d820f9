"""Pure-Python brute-force relational algebra on tiny relations (list of tuples).

Independent of oracle.c: used to pin it (tests/test_oracle_*.py).  Values are
python ints; typed wrap is done with explicit modular arithmetic here only
where a test needs it.
"""
from itertools import product

OPS = {
    "<": lambda x, y: x < y,
    "<=": lambda x, y: x <= y,
    ">": lambda x, y: x > y,
    ">=": lambda x, y: x >= y,
    "==": lambda x, y: x == y,
    "!=": lambda x, y: x != y,
}


def select(rows, preds):
    out = []
    for t in rows:
        ok = True
        for col, op, rhs in preds:
            y = t[rhs[1]] if isinstance(rhs, tuple) else rhs
            if not OPS[op](t[col], y):
                ok = False
        if ok:
            out.append(t)
    return out


def keep(rows, cols):
    return [tuple(t[c] for c in cols) for t in rows]


def nested_loop_join(L, R, nkey=1):
    """Definition: pairs with equal key, cross product of the value attributes,
    enumerated L-major then R — the order (key, iL, iR) for key-sorted inputs."""
    out = []
    for t in L:
        for u in R:
            if t[:nkey] == u[:nkey]:
                out.append(tuple(t) + tuple(u[nkey:]))
    return out


def group_sum(rows, gcols, gdomain, aggs):
    groups = {}
    for t in rows:
        g = tuple(t[c] for c in gcols)
        acc = groups.setdefault(g, [0] * (1 + len(aggs)))
        acc[0] += 1
        for k, a in enumerate(aggs):
            if a[0] == "sum":
                acc[1 + k] += t[a[1]]
    out = []
    for g in sorted(groups):
        acc = groups[g]
        row = list(g)
        for k, a in enumerate(aggs):
            row.append(acc[0] if a[0] == "count" else acc[1 + k])
        out.append(tuple(row))
    return out


def all_relations(max_n, ncols, values):
    """Every relation (ordered bag) with up to max_n rows over the given value set."""
    tuples = list(product(values, repeat=ncols))
    for n in range(max_n + 1):
        for rows in product(tuples, repeat=n):
            yield list(rows)


# ---------------------------------------------------------------------------
# A second, independent reader of the plan-spec format (oracle.evaluate is the
# first): every node evaluated with python ints, operator at a time, following the
# definitions of SURVEY §8(c) c1 and the readings of DESIGN.md §2 (A1 join output
# = key, left rest, right rest; A2 keep-list; A8 typed wrap; A10-A12 aggregates;
# A24 set operators on whole tuples).  Shares no code with oracle/.
# ---------------------------------------------------------------------------
WIDTH = {"i32": 32, "u32": 32, "i64": 64, "u64": 64, "u8": 8}
SIGNED = {"i32": True, "u32": False, "i64": True, "u64": False, "u8": False}


def wrap(t, v):
    """v reduced mod 2^w and read in type t (reading A8)."""
    w = WIDTH[t]
    v %= 1 << w
    if SIGNED[t] and v >= 1 << (w - 1):
        v -= 1 << w
    return v


def _expr(e, exprs, t_row, memo, i):
    if i in memo:
        return memo[i]
    x = exprs[i]
    op, typ = x[0], x[-1]
    if op == "col":
        v = wrap(typ, t_row[x[1]])
    elif op == "const":
        v = wrap(typ, x[1])
    elif op == "divc":
        a, k = wrap(typ, _expr(e, exprs, t_row, memo, x[1])), wrap(typ, x[2])
        q = abs(a) // abs(k)                      # truncation toward zero
        v = wrap(typ, q if (a >= 0) == (k >= 0) else -q)
    else:
        a = wrap(typ, _expr(e, exprs, t_row, memo, x[1]))
        b = wrap(typ, _expr(e, exprs, t_row, memo, x[2]))
        v = wrap(typ, a + b if op == "add" else a - b if op == "sub" else a * b)
    memo[i] = v
    return v


def project(rows, exprs, roots):
    out = []
    for t in rows:
        memo = {}
        out.append(tuple(_expr(None, exprs, t, memo, r) for r in roots))
    return out


def project_types(in_types, exprs, roots):
    return [exprs[r][-1] for r in roots]


def agg_rows(rows, gcols, gdomain, aggs):
    """(group codes..., then per aggregate: count, or the 128-bit sum as (lo u64, hi i64))."""
    groups = {}
    for t in rows:
        g = tuple(t[c] for c in gcols)
        for c, d in zip(g, gdomain):
            if not 0 <= c < d:
                raise ValueError("domain")
        acc = groups.setdefault(g, [0] * (1 + len(aggs)))
        acc[0] += 1
        for k, a in enumerate(aggs):
            if a[0] == "sum":
                acc[1 + k] += t[a[1]]
    out = []
    for g in sorted(groups):
        acc = groups[g]
        row = list(g)
        for k, a in enumerate(aggs):
            if a[0] == "count":
                row.append(acc[0])
            else:
                s = acc[1 + k] % (1 << 128)
                row += [s % (1 << 64), wrap("i64", s >> 64)]
        out.append(tuple(row))
    return out


def setop_rows(X, Y, op):
    sx, sy = set(X), set(Y)
    r = sx | sy if op == "union" else sx & sy if op == "intersect" else sx - sy
    return sorted(r)


def evaluate_spec(spec, inputs):
    """inputs: name -> list of tuples (python ints, in each column's type).
    Returns (types, rows) of spec["out"], every intermediate materialised."""
    env = {k: (list(v["types"]), list(inputs[k])) for k, v in spec["inputs"].items()}
    for nd in spec["nodes"]:
        op = nd["op"]
        if op == "select":
            types, rows = env[nd["in"]]
            preds = [(c, o, r if isinstance(r, tuple) else wrap(types[c], r)) for c, o, r in nd["preds"]]
            env[nd["id"]] = (types, select(rows, preds))
        elif op == "project":
            types, rows = env[nd["in"]]
            env[nd["id"]] = (project_types(types, nd["exprs"], nd["roots"]), project(rows, nd["exprs"], nd["roots"]))
        elif op == "join":
            k = nd.get("nkey", 1)
            (lt, lr), (rt, rr) = env[nd["left"]], env[nd["right"]]
            env[nd["id"]] = (lt + rt[k:], nested_loop_join(lr, rr, k))
        elif op in ("union", "intersect", "difference"):
            (xt, xr), (_, yr) = env[nd["left"]], env[nd["right"]]
            env[nd["id"]] = (xt, setop_rows(xr, yr, op))
        elif op == "agg":
            types, rows = env[nd["in"]]
            ot = [types[c] for c in nd["gcols"]]
            for a in nd["aggs"]:
                ot += ["i64"] if a[0] == "count" else ["u64", "i64"]
            env[nd["id"]] = (ot, agg_rows(rows, nd["gcols"], nd["gdomain"], nd["aggs"]))
        else:
            raise ValueError(op)
    return env[spec["out"]]
