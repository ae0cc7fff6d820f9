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
