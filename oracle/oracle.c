/*
 * oracle.c — plain, slow, obviously-correct CPU relational-algebra evaluator.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table or helper with the CUDA path (paper_conf_micro_wudcy12_b200/csrc).
 *
 * One operator at a time, every intermediate relation materialised in host
 * memory, single thread, no SIMD intrinsics.  Each function
 * cites the PAPER.md passage (P:<line>, section / table) whose definition it
 * writes out.  Readings of silent / garbled passages are the DESIGN.md
 * "Readings" table (A1..A23); the ones used here are named inline.
 *
 * Relation = bag of tuples of fixed-width integer attributes held as columns
 * (§2.2 "a relation is a set of tuples, each of which comprises of a list
 * of n attributes"; bag semantics per reading A3).
 *
 * Parity pins for every function live in tests/test_oracle_*.py.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_MAXCOLS 32

enum { OT_I32 = 0, OT_U32 = 1, OT_I64 = 2, OT_U64 = 3, OT_U8 = 4 };
enum { OC_LT = 0, OC_LE = 1, OC_GT = 2, OC_GE = 3, OC_EQ = 4, OC_NE = 5 };
enum { OE_COL = 0, OE_CONST = 1, OE_ADD = 2, OE_SUB = 3, OE_MUL = 4, OE_DIVC = 5 };
enum { OA_COUNT = 0, OA_SUM = 1 };

enum {
    OR_OK = 0,
    OR_E_ARG = -1,
    OR_E_TYPE = -2,
    OR_E_UNSORTED = -3,
    OR_E_DOMAIN = -4,
    OR_E_OOM = -5,
};

typedef struct {
    int64_t n;
    int32_t ncols;
    int32_t types[OR_MAXCOLS];
    void *cols[OR_MAXCOLS];
} orel;

typedef struct {            /* one atom of a conjunctive predicate (reading A4) */
    int32_t col;
    int32_t op;             /* OC_* */
    int32_t rhs_is_col;
    int32_t rhs_col;
    int64_t rhs_const;      /* converted to the column's type (wrap) */
} or_pred;

typedef struct {            /* expression node; explicit result type (reading A8) */
    int32_t op;             /* OE_* */
    int32_t type;           /* OT_I32/U32/I64/U64 */
    int32_t a, b;           /* child node indices (OE_COL: a = column index) */
    int64_t k;              /* OE_CONST value, OE_DIVC divisor */
} or_expr;

typedef struct {
    int32_t op;             /* OA_COUNT / OA_SUM */
    int32_t col;
} or_aggspec;

static int type_width(int t)
{
    switch (t) {
    case OT_I32: case OT_U32: return 4;
    case OT_I64: case OT_U64: return 8;
    case OT_U8: return 1;
    }
    return 0;
}

static int type_signed(int t) { return t == OT_I32 || t == OT_I64; }

/* Mathematical value of attribute (col, row) as a signed 128-bit integer. */
static __int128 get_value(const orel *r, int c, int64_t i)
{
    switch (r->types[c]) {
    case OT_I32: return ((const int32_t *)r->cols[c])[i];
    case OT_U32: return ((const uint32_t *)r->cols[c])[i];
    case OT_I64: return ((const int64_t *)r->cols[c])[i];
    case OT_U64: return ((const uint64_t *)r->cols[c])[i];
    case OT_U8: return ((const uint8_t *)r->cols[c])[i];
    }
    return 0;
}

/* Reduce a mathematical value into type t: mod 2^w, then read as signed or unsigned. */
static __int128 wrap_to(int t, __int128 v)
{
    switch (t) {
    case OT_I32: return (int32_t)(uint32_t)(unsigned __int128)v;
    case OT_U32: return (uint32_t)(unsigned __int128)v;
    case OT_I64: return (int64_t)(uint64_t)(unsigned __int128)v;
    case OT_U64: return (uint64_t)(unsigned __int128)v;
    case OT_U8: return (uint8_t)(unsigned __int128)v;
    }
    return 0;
}

static void put_value(orel *r, int c, int64_t i, __int128 v)
{
    switch (r->types[c]) {
    case OT_I32: ((int32_t *)r->cols[c])[i] = (int32_t)v; break;
    case OT_U32: ((uint32_t *)r->cols[c])[i] = (uint32_t)v; break;
    case OT_I64: ((int64_t *)r->cols[c])[i] = (int64_t)v; break;
    case OT_U64: ((uint64_t *)r->cols[c])[i] = (uint64_t)v; break;
    case OT_U8: ((uint8_t *)r->cols[c])[i] = (uint8_t)v; break;
    }
}

static int alloc_rel(orel *out, int64_t n, int ncols, const int32_t *types)
{
    memset(out, 0, sizeof(*out));
    out->n = n;
    out->ncols = ncols;
    for (int c = 0; c < ncols; c++) {
        out->types[c] = types[c];
        out->cols[c] = malloc((size_t)(n > 0 ? n : 1) * type_width(types[c]));
        if (!out->cols[c])
            return OR_E_OOM;
    }
    return OR_OK;
}

void or_free(orel *r)
{
    for (int c = 0; c < r->ncols; c++) {
        free(r->cols[c]);
        r->cols[c] = NULL;
    }
    r->ncols = 0;
    r->n = 0;
}

/* Shrink every column of `out` to its first `n` rows (the materialised size). */
static void set_rows(orel *out, int64_t n) { out->n = n; }

/* ------------------------------------------------------------------------ */
/* SELECT — P:104-107 Table 1: "consists of the set of tuples that satisfy a
 * predicate equation ... specified as a series of comparison operations on
 * tuple attributes".  Reading A4: conjunction of atoms, compared in the declared
 * column type; reading A5: input order preserved.                            */
/* ------------------------------------------------------------------------ */

static int compare(int op, __int128 x, __int128 y)
{
    switch (op) {
    case OC_LT: return x < y;
    case OC_LE: return x <= y;
    case OC_GT: return x > y;
    case OC_GE: return x >= y;
    case OC_EQ: return x == y;
    case OC_NE: return x != y;
    }
    return 0;
}

int or_select(const orel *in, int32_t npred, const or_pred *p, orel *out)
{
    for (int a = 0; a < npred; a++) {
        if (p[a].col < 0 || p[a].col >= in->ncols || p[a].op < 0 || p[a].op > OC_NE)
            return OR_E_ARG;
        if (p[a].rhs_is_col) {
            if (p[a].rhs_col < 0 || p[a].rhs_col >= in->ncols)
                return OR_E_ARG;
            if (in->types[p[a].rhs_col] != in->types[p[a].col])
                return OR_E_TYPE;
        }
    }
    int rc = alloc_rel(out, in->n, in->ncols, in->types);
    if (rc)
        return rc;
    int64_t m = 0;
    for (int64_t i = 0; i < in->n; i++) {
        int keep = 1;
        for (int a = 0; a < npred && keep; a++) {
            __int128 x = get_value(in, p[a].col, i);
            __int128 y = p[a].rhs_is_col ? get_value(in, p[a].rhs_col, i)
                                         : wrap_to(in->types[p[a].col], p[a].rhs_const);
            keep = compare(p[a].op, x, y);
        }
        if (keep) {
            for (int c = 0; c < in->ncols; c++)
                put_value(out, c, m, get_value(in, c, i));
            m++;
        }
    }
    set_rows(out, m);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* PROJECT with arithmetic — P:100-102 Table 1 ("after removing a specific set
 * of attributes"; example keeps [0,2] in order -> reading A2, keep-list in
 * output order), §4.3.1 (result is a new, narrower tuple), §4.4
 * (arithmetic +, -, x, / with thread dependence).  Reading A8: each expression
 * node carries its result type; operands are wrapped into it; +,-,x wrap mod
 * 2^w; DIVC truncates toward zero, divisor a nonzero constant, MIN/-1 wraps.  */
/* ------------------------------------------------------------------------ */

static __int128 eval_expr(const orel *in, const or_expr *e, int node, int64_t i)
{
    const or_expr *x = &e[node];
    __int128 a, b;
    switch (x->op) {
    case OE_COL:
        return wrap_to(x->type, get_value(in, x->a, i));
    case OE_CONST:
        return wrap_to(x->type, x->k);
    case OE_ADD:
        a = wrap_to(x->type, eval_expr(in, e, x->a, i));
        b = wrap_to(x->type, eval_expr(in, e, x->b, i));
        return wrap_to(x->type, a + b);
    case OE_SUB:
        a = wrap_to(x->type, eval_expr(in, e, x->a, i));
        b = wrap_to(x->type, eval_expr(in, e, x->b, i));
        return wrap_to(x->type, a - b);
    case OE_MUL:
        a = wrap_to(x->type, eval_expr(in, e, x->a, i));
        b = wrap_to(x->type, eval_expr(in, e, x->b, i));
        /* |a|,|b| < 2^64 so the product fits in 128 bits as unsigned; wrap after */
        return wrap_to(x->type, (__int128)((unsigned __int128)a * (unsigned __int128)b));
    case OE_DIVC: {
        a = wrap_to(x->type, eval_expr(in, e, x->a, i));
        b = wrap_to(x->type, x->k);
        /* C division on 128-bit truncates toward zero; MIN/-1 then wraps */
        return wrap_to(x->type, a / b);
    }
    }
    return 0;
}

static int check_expr(const orel *in, int32_t nexpr, const or_expr *e, int node, int depth)
{
    if (node < 0 || node >= nexpr || depth > 64)
        return OR_E_ARG;
    const or_expr *x = &e[node];
    if (x->type != OT_I32 && x->type != OT_U32 && x->type != OT_I64 && x->type != OT_U64) {
        if (!(x->op == OE_COL && x->type == OT_U8))
            return OR_E_TYPE;
    }
    switch (x->op) {
    case OE_COL:
        return (x->a >= 0 && x->a < in->ncols) ? OR_OK : OR_E_ARG;
    case OE_CONST:
        return OR_OK;
    case OE_ADD: case OE_SUB: case OE_MUL: {
        int rc = check_expr(in, nexpr, e, x->a, depth + 1);
        return rc ? rc : check_expr(in, nexpr, e, x->b, depth + 1);
    }
    case OE_DIVC:
        if (wrap_to(x->type, x->k) == 0)
            return OR_E_ARG;
        return check_expr(in, nexpr, e, x->a, depth + 1);
    }
    return OR_E_ARG;
}

int or_project(const orel *in, int32_t nexpr, const or_expr *e, int32_t nout,
               const int32_t *roots, orel *out)
{
    int32_t types[OR_MAXCOLS];
    if (nout < 0 || nout > OR_MAXCOLS)
        return OR_E_ARG;
    for (int j = 0; j < nout; j++) {
        int rc = check_expr(in, nexpr, e, roots[j], 0);
        if (rc)
            return rc;
        types[j] = e[roots[j]].type;
    }
    int rc = alloc_rel(out, in->n, nout, types);
    if (rc)
        return rc;
    for (int64_t i = 0; i < in->n; i++)
        for (int j = 0; j < nout; j++)
            put_value(out, j, i, eval_expr(in, e, roots[j], i));
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* JOIN — P:94-97 Table 1: "intersects on the key attribute and cross product
 * of value attributes" (reading A1: output = key, left non-key, right non-key;
 * the printed example output is an extraction loss).  Key = the leading nkey
 * attributes ("the 1st attribute is the key", reading A7).  Inputs are
 * key-sorted ("strict weak-ordering"); output ordered by (key, iL, iR)
 * (reading A5).  Plain two-pointer merge with nested loops over equal runs.  */
/* ------------------------------------------------------------------------ */

static int key_cmp(const orel *L, int64_t i, const orel *R, int64_t j, int nkey)
{
    for (int c = 0; c < nkey; c++) {
        __int128 x = get_value(L, c, i), y = get_value(R, c, j);
        if (x < y) return -1;
        if (x > y) return 1;
    }
    return 0;
}

static int is_sorted_on_key(const orel *r, int nkey)
{
    for (int64_t i = 1; i < r->n; i++)
        if (key_cmp(r, i - 1, r, i, nkey) > 0)
            return 0;
    return 1;
}

int or_join(const orel *L, const orel *R, int32_t nkey, orel *out)
{
    if (nkey < 1 || nkey > L->ncols || nkey > R->ncols)
        return OR_E_ARG;
    if (L->ncols + R->ncols - nkey > OR_MAXCOLS)
        return OR_E_ARG;
    for (int c = 0; c < nkey; c++)
        if (L->types[c] != R->types[c])
            return OR_E_TYPE;
    if (!is_sorted_on_key(L, nkey) || !is_sorted_on_key(R, nkey))
        return OR_E_UNSORTED;

    /* first pass: output size = sum over equal-key runs of lenL * lenR */
    int64_t total = 0;
    for (int64_t i = 0, j = 0; i < L->n && j < R->n;) {
        int c = key_cmp(L, i, R, j, nkey);
        if (c < 0) { i++; continue; }
        if (c > 0) { j++; continue; }
        int64_t i2 = i, j2 = j;
        while (i2 < L->n && key_cmp(L, i2, L, i, nkey) == 0) i2++;
        while (j2 < R->n && key_cmp(R, j2, R, j, nkey) == 0) j2++;
        total += (i2 - i) * (j2 - j);
        i = i2;
        j = j2;
    }

    int32_t types[OR_MAXCOLS];
    int nc = 0;
    for (int c = 0; c < L->ncols; c++) types[nc++] = L->types[c];
    for (int c = nkey; c < R->ncols; c++) types[nc++] = R->types[c];
    int rc = alloc_rel(out, total, nc, types);
    if (rc)
        return rc;

    int64_t m = 0;
    for (int64_t i = 0, j = 0; i < L->n && j < R->n;) {
        int c = key_cmp(L, i, R, j, nkey);
        if (c < 0) { i++; continue; }
        if (c > 0) { j++; continue; }
        int64_t i2 = i, j2 = j;
        while (i2 < L->n && key_cmp(L, i2, L, i, nkey) == 0) i2++;
        while (j2 < R->n && key_cmp(R, j2, R, j, nkey) == 0) j2++;
        for (int64_t a = i; a < i2; a++)
            for (int64_t b = j; b < j2; b++) {
                int oc = 0;
                for (int k = 0; k < L->ncols; k++)
                    put_value(out, oc++, m, get_value(L, k, a));
                for (int k = nkey; k < R->ncols; k++)
                    put_value(out, oc++, m, get_value(R, k, b));
                m++;
            }
        i = i2;
        j = j2;
    }
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* Group-by aggregate — P:43 §2.2 ("arithmetic computations ranging from
 * simple operators such as aggregation"), §5.2 TPC-H Q1.  Readings
 * A10-A12: group columns are dense codes with declared domains; COUNT is int64;
 * SUM is exact in 128 bits and returned as (lo u64, hi i64); only groups with
 * count > 0 are emitted, ascending group code g = sum code_c * stride_c where
 * the first group column varies slowest.  Out-of-domain code -> OR_E_DOMAIN.  */
/* ------------------------------------------------------------------------ */

int or_agg(const orel *in, int32_t ng, const int32_t *gcols, const int32_t *gdomain,
           int32_t na, const or_aggspec *a, orel *out)
{
    int64_t D = 1;
    if (ng < 0 || na < 0 || ng + 2 * na > OR_MAXCOLS)
        return OR_E_ARG;
    for (int c = 0; c < ng; c++) {
        if (gcols[c] < 0 || gcols[c] >= in->ncols || gdomain[c] < 1)
            return OR_E_ARG;
        D *= gdomain[c];
        if (D > (1 << 20))
            return OR_E_ARG;
    }
    for (int k = 0; k < na; k++)
        if ((a[k].op == OA_SUM && (a[k].col < 0 || a[k].col >= in->ncols)) ||
            (a[k].op != OA_SUM && a[k].op != OA_COUNT))
            return OR_E_ARG;

    int64_t *count = calloc((size_t)D, sizeof(int64_t));
    __int128 *sum = calloc((size_t)(D * (na > 0 ? na : 1)), sizeof(__int128));
    if (!count || !sum) {
        free(count);
        free(sum);
        return OR_E_OOM;
    }
    for (int64_t i = 0; i < in->n; i++) {
        int64_t g = 0;
        for (int c = 0; c < ng; c++) {
            __int128 code = get_value(in, gcols[c], i);
            if (code < 0 || code >= gdomain[c]) {
                free(count);
                free(sum);
                return OR_E_DOMAIN;
            }
            g = g * gdomain[c] + (int64_t)code;
        }
        count[g] += 1;
        for (int k = 0; k < na; k++)
            if (a[k].op == OA_SUM)
                sum[g * na + k] += get_value(in, a[k].col, i);
    }

    int64_t ngroups = 0;
    for (int64_t g = 0; g < D; g++)
        if (count[g] > 0)
            ngroups++;
    int32_t types[OR_MAXCOLS];
    int nc = 0;
    for (int c = 0; c < ng; c++) types[nc++] = in->types[gcols[c]];
    for (int k = 0; k < na; k++) {
        if (a[k].op == OA_COUNT) {
            types[nc++] = OT_I64;
        } else {
            types[nc++] = OT_U64;   /* lo */
            types[nc++] = OT_I64;   /* hi */
        }
    }
    int rc = alloc_rel(out, ngroups, nc, types);
    if (rc) {
        free(count);
        free(sum);
        return rc;
    }
    int64_t m = 0;
    for (int64_t g = 0; g < D; g++) {
        if (count[g] == 0)
            continue;
        int oc = 0;
        int64_t rem = g;
        /* decode g back into per-column codes (last column varies fastest) */
        int64_t codes[OR_MAXCOLS];
        for (int c = ng - 1; c >= 0; c--) {
            codes[c] = rem % gdomain[c];
            rem /= gdomain[c];
        }
        for (int c = 0; c < ng; c++)
            put_value(out, oc++, m, codes[c]);
        for (int k = 0; k < na; k++) {
            if (a[k].op == OA_COUNT) {
                put_value(out, oc++, m, count[g]);
            } else {
                unsigned __int128 u = (unsigned __int128)sum[g * na + k];
                put_value(out, oc++, m, (uint64_t)u);
                put_value(out, oc++, m, (int64_t)(uint64_t)(u >> 64));
            }
        }
        m++;
    }
    free(count);
    free(sum);
    return OR_OK;
}

/* Type helpers exported for the Python wrapper's self-checks. */
/* ------------------------------------------------------------------------ */
/* SET UNION / SET INTERSECTION / SET DIFFERENCE — P:69-83 Table 1: a new
 * relation "consisting of tuples ... present in at least one of the input
 * relations" (UNION), "present in both" (INTERSECTION), "exist in one input
 * relation and do not exist in the other" (DIFFERENCE, x minus y).  Reading
 * A24: membership is of the whole tuple (every attribute; the Table 1 examples
 * agree), set semantics (reading A3: the result has no duplicate tuples),
 * both inputs have identical schemas and are sorted on every attribute,
 * the result is ascending in that order (reading A5).
 * Plain definition: the distinct tuples of x ++ y in ascending order (a library
 * sort), each kept according to its membership in x and in y (a library binary
 * search in each sorted input).                                                */
/* ------------------------------------------------------------------------ */

enum { OS_UNION = 0, OS_INTERSECT = 1, OS_DIFFERENCE = 2 };

static const orel *g_sort_a, *g_sort_b;   /* qsort context: rows < a->n index a, else b */

static int row_cmp(const orel *A, int64_t i, const orel *B, int64_t j)
{
    return key_cmp(A, i, B, j, A->ncols);
}

static int cat_cmp(const void *pa, const void *pb)
{
    int64_t i = *(const int64_t *)pa, j = *(const int64_t *)pb;
    const orel *A = i < g_sort_a->n ? g_sort_a : g_sort_b;
    const orel *B = j < g_sort_a->n ? g_sort_a : g_sort_b;
    int64_t ii = i < g_sort_a->n ? i : i - g_sort_a->n;
    int64_t jj = j < g_sort_a->n ? j : j - g_sort_a->n;
    return row_cmp(A, ii, B, jj);
}

/* is row i of T a tuple of the sorted relation S? */
static int member(const orel *S, const orel *T, int64_t i)
{
    int64_t lo = 0, hi = S->n;
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        int c = row_cmp(S, mid, T, i);
        if (c == 0) return 1;
        if (c < 0) lo = mid + 1;
        else hi = mid;
    }
    return 0;
}

int or_setop(const orel *X, const orel *Y, int32_t op, orel *out)
{
    if (op < OS_UNION || op > OS_DIFFERENCE || X->ncols != Y->ncols || X->ncols < 1)
        return OR_E_ARG;
    for (int c = 0; c < X->ncols; c++)
        if (X->types[c] != Y->types[c])
            return OR_E_TYPE;
    if (!is_sorted_on_key(X, X->ncols) || !is_sorted_on_key(Y, Y->ncols))
        return OR_E_UNSORTED;
    const int64_t n = X->n + Y->n;
    int64_t *idx = (int64_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));
    if (!idx)
        return OR_E_OOM;
    for (int64_t i = 0; i < n; i++)
        idx[i] = i;
    g_sort_a = X;
    g_sort_b = Y;
    qsort(idx, (size_t)n, sizeof(int64_t), cat_cmp);
    /* distinct tuples, ascending; keep per membership */
    int64_t *keep = (int64_t *)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));
    if (!keep) {
        free(idx);
        return OR_E_OOM;
    }
    int64_t m = 0;
    for (int64_t q = 0; q < n; q++) {
        if (q > 0 && cat_cmp(&idx[q - 1], &idx[q]) == 0)
            continue;                                   /* duplicate tuple */
        const orel *T = idx[q] < X->n ? X : Y;
        const int64_t r = idx[q] < X->n ? idx[q] : idx[q] - X->n;
        const int inx = member(X, T, r), iny = member(Y, T, r);
        const int k = op == OS_UNION ? (inx || iny) : op == OS_INTERSECT ? (inx && iny) : (inx && !iny);
        if (k)
            keep[m++] = idx[q];
    }
    int rc = alloc_rel(out, m, X->ncols, X->types);
    if (rc == OR_OK)
        for (int64_t q = 0; q < m; q++) {
            const orel *T = keep[q] < X->n ? X : Y;
            const int64_t r = keep[q] < X->n ? keep[q] : keep[q] - X->n;
            for (int c = 0; c < X->ncols; c++)
                put_value(out, c, q, get_value(T, c, r));
        }
    free(idx);
    free(keep);
    return rc;
}

int or_type_width(int t) { return type_width(t); }
int or_type_signed(int t) { return type_signed(t); }
