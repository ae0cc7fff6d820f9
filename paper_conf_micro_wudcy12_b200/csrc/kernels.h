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

struct JoinRunsLaunch {
    const void *lkey, *rkey;
    int64_t nl, nr;
    int64_t nparts;
    uint32_t *s, *lenL, *lo, *lenR;
    uint64_t *off;
    int64_t cap_runs;
    uint64_t *status_runs, *status_outs;
    uint32_t epoch_runs, epoch_outs;
    uint32_t *ctrs;
    int64_t *totals;                 // [0] runs, [1] join candidates
    int64_t *split;                  // nparts + 1 merge-path splits (k_merge_splits)
    uint64_t *pruns, *pouts;         // per-partition counts, then exclusive offsets
    // SELECTs on the join key fused into the run matching (SURVEY §8(f) N2
    // Fig. 13): a run is matched only if its key passes every atom (key op kpk[i]),
    // compared in the key type; a key predicate keeps or drops whole runs
    int32_t nkpred;
    uint8_t kop[kMaxKeyPreds];
    int64_t kpk[kMaxKeyPreds];
};

struct JoinExpand {
    const uint32_t *s, *lo, *lenR;
    const uint64_t *off;
    const int64_t *tile_run;
    int64_t nruns;
    int32_t ncols;                   // gathered (live) join output columns
    const void *src[kMaxSlots];
    uint8_t from_right[kMaxSlots];
    int16_t dst_slot[kMaxSlots];
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
size_t join_run_cache_bytes();
int chain_occupancy(int which, int nt, int items, size_t smem);   // which: 0 scan, 1 scan+agg, 2 join expand, 3 join runs, 4 scan branches
cudaError_t scan_chain_launch(const ChainProg &P, const TileLaunch &L, bool agg, int nt, int items, size_t smem, int grid,
                              cudaStream_t s);
cudaError_t agg_finalize_launch(const AggFinal &F, cudaStream_t s);
cudaError_t join_runs_launch(const JoinRunsLaunch &J, int key_type, size_t smem, int grid, cudaStream_t s);
size_t join_runs_smem(int key_type);
cudaError_t tile_runs_launch(const uint64_t *off, int64_t nruns, int64_t ntiles, int64_t T, int64_t *tile_run,
                             cudaStream_t s);
int join_expand_tile();
cudaError_t join_chain_launch(const ChainProg &P, const TileLaunch &L, const JoinExpand &X, size_t smem, int grid,
                              cudaStream_t s);
int scan_tile();

// emitting scan kernel (scan_emit.cu): compacting SELECT / PROJECT chains, 1..4 branches
size_t emit_ctl_bytes();
int scan_emit_occupancy(int nt, int items, bool multi, size_t smem);
cudaError_t scan_emit_launch(const ChainProg &P, const TileLaunch &L, int nt, int items, size_t smem, int grid,
                             cudaStream_t s);

}  // namespace rw
