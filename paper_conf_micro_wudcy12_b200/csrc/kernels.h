// kernels.h — host-side launch interface of the sm_100a kernels (internal).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include "internal.h"

namespace rw {

constexpr int kMaxStages = 8;
constexpr int kMaxKeyPreds = 8;      // key-predicate atoms fused into one JOIN

struct AggFinal {
    const unsigned long long *acc;   // D * NA * 2 (lo, hi); zeroed by the finalize kernel after reading
    unsigned long long *acc_w;       // same pointer, writable
    int32_t D, NA, ngc;
    int32_t gdomain[kMaxGroupCols];
    uint8_t gtype[kMaxGroupCols];
    int32_t nreq;                    // requested aggregates in output order
    uint8_t req_is_sum[kMaxAggs];
    int16_t req_acc[kMaxAggs];       // accumulator index a (0 = count)
    void *out[kMaxOut];
    int64_t capacity;
    int64_t *n_dev;
    int32_t *err;                    // err[0] -> err[1], err[2] -> err[3], then err[0] = err[2] = 0
};

// set operators (setops.cu): inputs sorted on every column, identical schemas
constexpr int kMaxSetCols = 4;
struct SetLaunch {
    int32_t ncols;
    int32_t op;                      // 0 UNION, 1 INTERSECT, 2 DIFFERENCE (x - y)
    uint8_t types[kMaxSetCols];
    const void *x[kMaxSetCols], *y[kMaxSetCols];
    void *out[kMaxSetCols];
    int64_t nx, ny, nparts, cap;
    int64_t *split;                  // nparts + 1 merge-path splits
    int32_t *nbr;                    // per split: has_pred | pred_is_x << 1 | has_succ << 2 | succ_is_x << 3
    uint64_t *pcount;                // per-partition emitted rows, then exclusive offsets
    int64_t *total;                  // device row count of the result
    uint64_t *status;                // non-null: single pass with decoupled look-back (nparts words)
    uint32_t epoch;
    uint32_t *ctrs;                  // single pass: [0] partition counter, [1] exit counter (reset by the last CTA)
};
size_t set_op_smem(int ncols);
int set_partition_rows();
cudaError_t set_op_launch(const SetLaunch &S, int sms, cudaStream_t st);   // 2 launches (look-back) or 4

size_t scan_ctl_bytes();
int chain_occupancy(int which, int nt, int items, size_t smem);   // which: 0 scan, 1 scan+agg, 4 scan branches
cudaError_t scan_chain_launch(const ChainProg &P, const TileLaunch &L, bool agg, int nt, int items, size_t smem, int grid,
                              cudaStream_t s);
cudaError_t agg_finalize_launch(const AggFinal &F, cudaStream_t s);


int scan_tile();

// ---- join2.cu: run matching (single pass) and the fused expansion ----
struct KeySrc {                      // order-preserving image of the leading nkey (<= 2) key columns
    const void *col[2];
    uint8_t type[2];
    int32_t ncol;
    const void *img;                 // non-null: precomputed images (uint32 / uint64 array)
};

struct MatchLaunch {
    KeySrc A, B;
    int64_t nA, nB, nparts;          // nparts: launched partitions (an upper bound when nA_dev is set)
    const int64_t *nA_dev;           // chained match: A's row count on the device (else null: nA)
    int64_t *split;                  // nparts + 1 merge-path splits
    const uint64_t *wA;              // chained match: weight of every A element (first-level run), else null
    // chained (3-input) composition: A element ga = first-level run, whose (s0, s1, len1) are copied
    int32_t chain1;
    const uint32_t *c_s0, *c_s1, *c_len1;
    // outputs: one record per matched key, in key order (capacity cap_runs + 8 padded)
    uint32_t *s0, *s1, *len1, *s2, *len2, *len0;
    void *key_out;                   // optional key images of the runs (chaining)
    uint64_t *w_out;                 // optional lenA * lenB per run (chaining)
    uint64_t *off;                   // exclusive prefix of the runs' candidate counts
    int64_t cap_runs;
    uint64_t *st_runs, *st_cands;    // look-back status words, nparts each
    uint32_t ep_runs, ep_cands;
    uint32_t *ctrs;
    int64_t *totals;                 // [0] runs, [1] candidates
    int32_t nkpred;                  // fused key SELECT atoms (N2): on the key image
    uint8_t kop[kMaxKeyPreds];
    uint64_t kpk[kMaxKeyPreds];
};

struct JoinEmit {
    const int64_t *tile_run;         // first run of every tile (+ entry ntiles = nruns - 1)
    const uint64_t *off;
    const uint32_t *s0, *s1, *len1, *s2, *len2;
    uint32_t rec_cap4, rec_stage_bytes;
    int32_t ncols;                   // live join columns gathered into input slots 0..ncols-1
    const void *src[kMaxSlots];
    uint8_t w[kMaxSlots];
    uint8_t side[kMaxSlots];         // 0: first input (row s0 + i), 1: second (s1 + j), 2: third (s2 + k)
    int32_t regpath;                 // gathers through registers (<= 4 live columns, all 1 or 4 bytes)
};

int match_partition();
cudaError_t match_launch(const MatchLaunch &M, bool wide, cudaStream_t st);
cudaError_t jtiles_launch(const uint64_t *off, const int64_t *totals, int64_t T, int64_t cap_tiles, int64_t *tile_run,
                          int32_t *overflow, int sms, cudaStream_t st);
uint32_t join_rec_cap4(int T);
size_t join_rec_stage_bytes(int ways, int T);
size_t join_emit_ctl_bytes();
int join_emit_occupancy(int nt, int items, int ways, size_t smem, bool agg);
cudaError_t join_emit_launch(const ChainProg &P, const TileLaunch &L, const JoinEmit &X, int nt, int items, int ways,
                             size_t smem, int grid, cudaStream_t s);

// emitting scan kernel (scan_emit.cu): compacting SELECT / PROJECT chains, 1..4 branches
size_t emit_ctl_bytes();
int scan_emit_occupancy(int nt, int items, bool multi, size_t smem, int teams = 1);
cudaError_t scan_emit_launch(const ChainProg &P, const TileLaunch &L, int nt, int items, size_t smem, int grid,
                             cudaStream_t s, int teams = 1);

}  // namespace rw
