// dist_kernels.h — host launch interface of the multi-GPU helper kernels (internal).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace rw {

constexpr int kMaxMergeCols = 8;

struct MergeCols {
    const void *col[kMaxMergeCols];
};
struct MergeOut {
    void *col[kMaxMergeCols];
};
struct MergeTypes {
    uint8_t t[kMaxMergeCols];
};

// Aggregate relation <-> dense limbs.  Per group g (D of them) L int64 words:
// [presence] then per requested aggregate: COUNT -> 1 word, SUM -> 4 limbs of 32 bits
// (two's complement 128-bit value), so an int64 sum over <= 2^31 ranks is exact.
struct AggXfer {
    const void *col[kMaxOut];       // export: local aggregate output columns
    int32_t ngc;
    int32_t gdomain[kMaxGroupCols];
    uint8_t gtype[kMaxGroupCols];
    int32_t nreq;
    uint8_t is_sum[kMaxAggs];
    int32_t D;
    int32_t L;
};

struct OutPtrs {
    void *col[kMaxOut];
};

// Single-pass P-way merge (merge_p.cu).  Runs lie at rows [run_off[q], run_off[q+1])
// of every column (or of `packed`, u64 order-preserving tuple images); T = sample
// spacing, G = samples per merge group, S = samples, NG = groups.
constexpr int kMpThreads = 256;
constexpr int kMpItems = 16;
constexpr int kMpC = kMpThreads * kMpItems;   // elements one merge group may hold
constexpr int kMpCP = kMpC + kMpC / 16;      // shared-memory words of one buffer (padded)
constexpr int kMpMaxRuns = 32;

struct MpLaunch {
    const void *col[kMaxMergeCols];
    uint8_t types[kMaxMergeCols];
    int32_t ncols;
    const uint64_t *packed;              // packed u64 input (else nullptr: read col[])
    int32_t nrun;
    int32_t T;
    int32_t G;
    int64_t run_off[kMpMaxRuns + 1];
    int64_t samp_base[kMpMaxRuns + 1];
    int64_t S;
    int64_t NG;
    uint64_t *sv;                        // S sample images
    uint32_t *cuts;                      // NG x nrun: cut of every run at every group start
    int64_t *bound;                      // NG group-start samples
    void *out[kMaxMergeCols];
};

cudaError_t mp_merge_launch(const MpLaunch &M, int sms, cudaStream_t s);
cudaError_t mp_pack_launch(const MpLaunch &M, int64_t n, uint64_t *dst, int sms, cudaStream_t s);

cudaError_t split_bounds_launch(const void *keys, int64_t n, int key_type, const void *spl, int nsplit,
                                int64_t *bounds, cudaStream_t s);
cudaError_t merge2_launch(const MergeCols &A, int64_t na, const MergeCols &B, int64_t nb, const MergeOut &O,
                          int ncols, const MergeTypes &T, cudaStream_t s);
cudaError_t agg_export_launch(const AggXfer &X, const int64_t *n_dev, int64_t n_host, int64_t *limbs,
                              cudaStream_t s);
cudaError_t agg_import_launch(const AggXfer &X, const int64_t *limbs, const OutPtrs &out, int64_t cap,
                              int64_t *n_dev, cudaStream_t s);

}  // namespace rw
