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

cudaError_t split_bounds_launch(const void *keys, int64_t n, int key_type, const void *spl, int nsplit,
                                int64_t *bounds, cudaStream_t s);
cudaError_t merge2_launch(const MergeCols &A, int64_t na, const MergeCols &B, int64_t nb, const MergeOut &O,
                          int ncols, const MergeTypes &T, cudaStream_t s);
cudaError_t agg_export_launch(const AggXfer &X, const int64_t *n_dev, int64_t n_host, int64_t *limbs,
                              cudaStream_t s);
cudaError_t agg_import_launch(const AggXfer &X, const int64_t *limbs, const OutPtrs &out, int64_t cap,
                              int64_t *n_dev, cudaStream_t s);

}  // namespace rw
