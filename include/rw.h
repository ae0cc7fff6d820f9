/*
 * rw.h — C ABI of the fused relational-algebra engine (librw.so), sm_100a.
 *
 * What it computes: a query plan (DAG) of relational-algebra operators over
 * fixed-width integer / fixed-point tuples, executed as fused groups — the hot
 * path of Kernel Weaver (Wu, Diamos, Cadambi, Yalamanchili, MICRO'12).
 * Citations: "P:<line>" = /root/reference/PAPER.md line, with its section /
 * table.  "A<n>" = the paper readings listed in DESIGN.md ("Readings").
 *
 * Data model (§2.2, §3): a relation is a bag of tuples (A3) of
 * fixed-width integer attributes.  The library stores it column-wise: one
 * DEVICE array per attribute, row i of every column forming tuple i.
 *
 * Ownership: every pointer passed in is owned by the caller.  Device pointers
 * must stay valid until the work enqueued on the plan's stream completes.
 * Scratch owned by the plan (look-back status words, tile counters, run
 * records, intermediates at kernel-dependence boundaries) is allocated with
 * cudaMallocAsync on the plan's stream and released by rw_plan_destroy.
 *
 * Errors: every call returns rw_status (0 = RW_OK, negative = error).  No C++
 * exception crosses the ABI.  On error the outputs are untouched unless stated.
 * rw_last_error() returns a thread-local message for the last failure.  After
 * RW_E_CUDA the plan must be destroyed.  A plan is not thread-safe.
 * There is no CPU fallback: without a usable sm_100 device, rw_plan_create
 * fails with RW_E_CUDA.
 */
#ifndef RW_H
#define RW_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t rw_status;
#define RW_OK 0
#define RW_E_ARG (-1)          /* bad argument / node id / column index */
#define RW_E_TYPE (-2)         /* type mismatch (col-vs-col atom, join key, group column) */
#define RW_E_UNSORTED (-3)     /* JOIN input not declared sorted on the join key (A6) */
#define RW_E_OVERFLOW (-4)     /* strict mode: i64/u64 expression may wrap (A8) */
#define RW_E_UNSUPPORTED (-5)  /* outside what this build implements (e.g. nkey > 2) */
#define RW_E_CAPACITY (-6)     /* output capacity too small; required rows in out->n */
#define RW_E_OOM (-7)
#define RW_E_CUDA (-8)
#define RW_E_DOMAIN (-9)       /* AGG: a group column value outside [0, domain) */
#define RW_E_STATE (-10)

/* Attribute types (A8: i32/u32 wrap mod 2^32; fixed point = I64 with a decimal scale
 * chosen by the caller, e.g. DECIMAL(15,2) stored as cents). */
typedef enum { RW_I32 = 0, RW_U32 = 1, RW_I64 = 2, RW_U64 = 3, RW_U8 = 4 } rw_type;

/* Comparison of a SELECT atom (Table 1 "a series of comparison operations on
 * tuple attributes"; A4: conjunction of atoms, compared in the column's type). */
typedef enum { RW_LT = 0, RW_LE = 1, RW_GT = 2, RW_GE = 3, RW_EQ = 4, RW_NE = 5 } rw_cmp;

/* Expression node of a PROJECT (Table 1, §4.3.1, §4.4). */
typedef enum { RW_COL = 0, RW_CONST = 1, RW_ADD = 2, RW_SUB = 3, RW_MUL = 4, RW_DIVC = 5 } rw_expr_op;

typedef enum { RW_COUNT = 0, RW_SUM = 1 } rw_agg_op;

/* Set operators (Table 1). */
typedef enum { RW_UNION = 0, RW_INTERSECT = 1, RW_DIFFERENCE = 2 } rw_setop;

/* One SELECT atom: (col OP rhs).  rhs = column rhs_col (same type as col, else
 * RW_E_TYPE) when rhs_is_col, else rhs_const reduced mod 2^w into col's type. */
typedef struct {
    int32_t col;
    int32_t op;        /* rw_cmp */
    int32_t rhs_is_col;
    int32_t rhs_col;
    int64_t rhs_const;
} rw_pred;

/* Expression node.  `type` is the node's result type (RW_I32/U32/I64/U64; RW_U8 only
 * for RW_COL).  Operands are converted into `type` (mod 2^w), then
 *   RW_COL  : input column a                 RW_CONST: constant k
 *   RW_ADD/SUB/MUL: nodes a, b (earlier indices), wrapping mod 2^w
 *   RW_DIVC : node a / k, k != 0, truncation toward zero, MIN / -1 = MIN. */
typedef struct {
    int32_t op;        /* rw_expr_op */
    int32_t type;      /* rw_type */
    int32_t a;
    int32_t b;
    int64_t k;
} rw_expr;

/* Aggregate: RW_COUNT (col ignored) -> one I64 output column; RW_SUM of column col
 * -> two output columns (lo: U64, hi: I64) holding the exact 128-bit sum
 * hi * 2^64 + lo (A11). */
typedef struct {
    int32_t op;        /* rw_agg_op */
    int32_t col;
} rw_agg;

typedef struct {
    int32_t device;           /* CUDA device ordinal */
    void *cuda_stream;        /* cudaStream_t all work is enqueued on; NULL = legacy default */
    int32_t fuse;             /* 1: fuse thread/CTA-dependent operators (§4.1);
                                 0: operator-at-a-time, every intermediate materialised */
    int32_t zero_copy_project;/* fuse == 0 only: a PROJECT of plain column references
                                 aliases its input columns instead of copying */
    int32_t stages;           /* 0 = auto: TMA tiles in flight per CTA (1..8) */
    int32_t ctas_per_sm;      /* 0 = auto (occupancy) */
    int32_t strict_overflow;  /* 1: reject i64/u64 expressions whose interval may wrap */
    int32_t host_chunk_log2;  /* rw_plan_execute_host: rows per streamed chunk = 2^this
                                 (0 = auto, 2^25) */
    int32_t reserved[8];
} rw_plan_opts;

typedef struct rw_plan rw_plan;

/* Input relations of one execute: row count and one device pointer per column,
 * in the schema order given to rw_plan_add_input.  Column bases should be 16-byte
 * aligned (TMA bulk staging); unaligned bases take a slower load path. */
typedef struct {
    int64_t n;
    const void *const *cols;
} rw_relation_in;

/* Output of one execute.  cols: one caller-owned device buffer per output column,
 * each holding `capacity` rows.  If n_dev != NULL the row count is written there
 * asynchronously and execute returns without synchronising (n = -1; rows beyond
 * capacity are dropped and the caller compares *n_dev with capacity).  If
 * n_dev == NULL execute synchronises the stream and sets n; n > capacity returns
 * RW_E_CAPACITY (n = required rows, buffer holds the first `capacity`). */
typedef struct {
    void **cols;
    int64_t capacity;
    int64_t *n_dev;
    int64_t n;
} rw_relation_out;

/* ---- plan construction (host only, no device work) ---------------------- */

rw_status rw_plan_create(rw_plan **out, const rw_plan_opts *opts);
void rw_plan_destroy(rw_plan *plan);

/* Declare an input relation: ncols attribute types; nkey_sorted = number of leading
 * columns the data is sorted on (lexicographic, ascending in each type; 0 = unsorted;
 * A6).  lo/hi (optional, NULL = full type range): caller-promised inclusive value
 * bounds per column, used by interval analysis (aggregate flush period, strict mode).
 * The bounds are a correctness precondition of the aggregate terminal: sums of columns
 * declared within [0, 2^16) accumulate in 32-bit partials flushed on a period derived
 * from the bounds.  A summed narrow value outside [0, 2^b) (b = bits of the declared
 * upper bound) is detected and reported as RW_E_DOMAIN by the execute that finalises
 * the aggregate; wide sums keep 64-bit partials flushed before they could overflow
 * under the declared bounds (undefined sums if data exceed them by orders of magnitude). */
rw_status rw_plan_add_input(rw_plan *plan, int32_t ncols, const int32_t *types, int32_t nkey_sorted,
                            const int64_t *lo, const int64_t *hi, int32_t *node);

/* SELECT: conjunction of np atoms over node `in`; schema and order kept. */
rw_status rw_plan_add_select(rw_plan *plan, int32_t in, const rw_pred *p, int32_t np, int32_t *node);

/* PROJECT: nout output columns, output j = expression
 * tree rooted at e[roots[j]] over node `in`'s columns (A2: keep-list in order). */
rw_status rw_plan_add_project(rw_plan *plan, int32_t in, const rw_expr *e, int32_t ne,
                              const int32_t *roots, int32_t nout, int32_t *node);

/* JOIN (A1): equi-join on the leading nkey columns (this build: nkey == 1;
 * else RW_E_UNSUPPORTED).  Both inputs must be sorted on the key (RW_E_UNSORTED) with
 * identical key types (RW_E_TYPE).  Output schema = (key, left non-key..., right
 * non-key...), rows ordered by (key, left row, right row) (A5). */
rw_status rw_plan_add_join(rw_plan *plan, int32_t left, int32_t right, int32_t nkey, int32_t *node);

/* SET UNION / SET INTERSECTION / SET DIFFERENCE (Table 1; reading A24):
 * membership of whole tuples, set semantics (the result has no duplicate tuple even
 * if an input has), RW_DIFFERENCE = left minus right.  Both inputs need identical
 * schemas (RW_E_TYPE) of at most 4 columns (RW_E_UNSUPPORTED) and must be sorted on
 * every column, lexicographically in the declared signedness (nkey_sorted == ncols,
 * else RW_E_UNSORTED).  Output: same schema, ascending, sorted on every column.
 * Runs as a merge-path kernel with a decoupled look-back over the materialised inputs
 * (SURVEY §8(f) N3); a downstream SELECT / PROJECT scans its output. */
rw_status rw_plan_add_setop(rw_plan *plan, int32_t left, int32_t right, int32_t op, int32_t *node);

/* Group-by aggregate (§2.2, §5.2 Q1; A10-A12): group columns are dense
 * codes 0 <= v < gdomain[c] (prod of domains <= 4096, else RW_E_UNSUPPORTED).  Output:
 * group columns (input types), then per aggregate its column(s) (see rw_agg).  Only
 * groups with at least one row, ascending code with the first group column slowest. */
rw_status rw_plan_add_agg(rw_plan *plan, int32_t in, const int32_t *gcols, const int32_t *gdomain,
                          int32_t ng, const rw_agg *a, int32_t na, int32_t *node);

/* Output schema of a node: *ncols and types[0..ncols) (types may be NULL; cap 32). */
rw_status rw_plan_node_schema(const rw_plan *plan, int32_t node, int32_t *ncols, int32_t *types);

/* ---- execution ---------------------------------------------------------- */

/* Execute the plan for node out_node.  in[i] supplies the i-th declared input
 * (declaration order).  Enqueues every kernel on the plan's stream.  Plans whose
 * path contains a JOIN synchronise once per JOIN (after the run-count phase) to size
 * the expansion. */
rw_status rw_plan_execute(rw_plan *plan, const rw_relation_in *in, int32_t nin, int32_t out_node,
                          rw_relation_out *out);

/* Input-dependence fusion (§4.4 "operators shares the same inputs ... the input
 * data shared by different operators only need to be loaded once"; Fig. 14(d)):
 * execute nout output nodes at once.  outs[k] receives out_nodes[k] exactly as
 * rw_plan_execute would (same layout, capacity and n / n_dev rules, same row order).
 * When the plan is fused, 2 <= nout <= 4, and every out_nodes[k] is reached from one
 * common INPUT relation through SELECT / PROJECT nodes only, all branches run in ONE
 * k_scan_chain pass: each tile is loaded once and every branch evaluates, compacts and
 * stores its own output.  Otherwise (fuse = 0, other shapes) the nodes run one after
 * the other, each as rw_plan_execute.  A shared SELECT/PROJECT prefix of several
 * branches is re-evaluated per branch (thread-dependent work, no extra bytes).
 * Errors as rw_plan_execute; RW_E_CAPACITY names the first output that overflowed. */
rw_status rw_plan_execute_multi(rw_plan *plan, const rw_relation_in *in, int32_t nin, const int32_t *out_nodes,
                                int32_t nout, rw_relation_out *outs);

/* Same, with HOST buffers: inputs are copied host->device, the plan runs, the result
 * (up to capacity rows) is copied device->host, the stream is synchronised and out->n
 * set.  Pinned (cudaHostAlloc / registered) buffers give full PCIe bandwidth.
 * Host streaming (the paper's PCIe experiment, §5.1.3): when the plan is
 * one fused scan group over one INPUT relation (SELECT / PROJECT / arithmetic chain,
 * optionally ending in an AGG) and the input exceeds one chunk (opts.host_chunk_log2),
 * it runs chunk by chunk with the H2D copy of chunk k+1, the kernel of chunk k and the
 * D2H copy of chunk k-1's compacted rows overlapped on three streams (double-buffered
 * device chunks, allocated per call).  The result is identical to the unchunked run,
 * row order included; an aggregate accumulates every chunk and finalises once.
 * Other plans copy the whole inputs first. */
rw_status rw_plan_execute_host(rw_plan *plan, const rw_relation_in *in, int32_t nin, int32_t out_node,
                               rw_relation_out *out);

/* Human-readable fusion report: groups, edge classes (thread / CTA / kernel, P:156-164
 * §4.1 Fig. 8), kernel template and resource estimate per group (Alg. 1/2 analogue,
 * P:164-171).  Writes at most cap bytes (NUL-terminated); returns RW_OK or
 * RW_E_CAPACITY when truncated. */
rw_status rw_plan_explain(rw_plan *plan, int32_t out_node, char *buf, size_t cap);

/* Number of sm_100a kernels the last execute launched (memsets excluded). */
int64_t rw_plan_last_launches(const rw_plan *plan);

const char *rw_status_str(rw_status s);
const char *rw_last_error(void);

/* ---- multi-GPU helpers (row / key-range sharding) ---------- */

/* Key-range split of a key-sorted column: for each of the nsplit ascending splitter
 * values, the number of rows with key < splitter (lower bound), written to
 * bounds_dev[0..nsplit) (device int64).  key_type is rw_type of the column. */
rw_status rw_split_by_splitters(const void *keys_dev, int64_t n, int32_t key_type, const void *splitters_dev,
                                int32_t nsplit, int64_t *bounds_dev, void *cuda_stream);

/* Merge nrun runs, each sorted lexicographically over all ncols columns (<= 8), that
 * lie concatenated in `cols` (run r = rows [run_off[r], run_off[r+1]) of every column;
 * run_off is a HOST array of nrun+1 entries) into one sequence sorted the same way,
 * written to out_cols (device, run_off[nrun] - run_off[0] rows).  Equal tuples keep run
 * order.  This is the merge after the key-range all-to-all (§4.3.2
 * merge-path partitioning generalised to P inputs).  Tuples of <= 8 bytes with 2 <=
 * nrun <= 32: one pass (read once, write once; merge_p.cu), each run < 2^32 rows, else
 * RW_E_UNSUPPORTED.  Wider tuples or more runs: pairwise merge-path tree
 * (ceil(log2 nrun) passes).  Temporaries come from cudaMallocAsync on the stream. */
rw_status rw_merge_runs(const void *const *cols, const int32_t *types, int32_t ncols, const int64_t *run_off,
                        int32_t nrun, void *const *out_cols, void *cuda_stream);

/* Order-preserving u64 image of each of n tuples whose columns total <= 8 bytes
 * (columns concatenated, first column most significant, signed types with the sign bit
 * flipped), so that u64 order = lexicographic tuple order in the declared types; written
 * to packed_dev[0..n).  The exchange sends these images in ONE all-to-all instead of one
 * per column.  Tuples wider than 8 bytes: RW_E_UNSUPPORTED. */
rw_status rw_pack_tuples(const void *const *cols, const int32_t *types, int32_t ncols, int64_t n,
                         uint64_t *packed_dev, void *cuda_stream);

/* rw_merge_runs over runs of packed images (rw_pack_tuples layout): run r = entries
 * [run_off[r], run_off[r+1]) of packed_dev (run_off on the HOST, nrun <= 32, each run
 * < 2^32 rows); the merged tuples are unpacked into the ncols device columns out_cols
 * (run_off[nrun] - run_off[0] rows).  One read and one write pass. */
rw_status rw_merge_packed_runs(const uint64_t *packed_dev, const int32_t *types, int32_t ncols,
                               const int64_t *run_off, int32_t nrun, void *const *out_cols, void *cuda_stream);

/* Aggregate combine across row shards: an aggregate result is
 * exported as D * L dense int64 words (per group: a presence word, then per aggregate
 * 1 word for COUNT or four 32-bit limbs of the 128-bit two's complement SUM), so that a
 * plain int64 SUM all-reduce over <= 2^31 ranks is exact; import recombines the limbs
 * (sum_k limb_k * 2^32k mod 2^128) and emits the groups present on any rank, ascending.
 * rw_plan_agg_limbs gives D * L.  export: cols = the node's local result columns on
 * device, row count from n_dev (device) or n_host; limbs_dev is overwritten.  Both are
 * enqueued on the plan's stream; import synchronises when out->n_dev is NULL. */
rw_status rw_plan_agg_limbs(const rw_plan *plan, int32_t agg_node, int64_t *nlimbs);
rw_status rw_plan_agg_export(rw_plan *plan, int32_t agg_node, const void *const *cols, const int64_t *n_dev,
                             int64_t n_host, int64_t *limbs_dev);
rw_status rw_plan_agg_import(rw_plan *plan, int32_t agg_node, const int64_t *limbs_dev, rw_relation_out *out);

#ifdef __cplusplus
}
#endif
#endif /* RW_H */
