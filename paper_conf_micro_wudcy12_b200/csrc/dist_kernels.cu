// dist_kernels.cu — sm_100a kernels for multi-GPU sharding:
//   k_split_bounds   key-range split of a key-sorted column by splitter values
//   k_merge2         stable merge-path merge of two sorted runs (lexicographic over
//                    all columns); rw_merge_runs builds a P-way merge tree from it
//   k_agg_export     local aggregate relation -> dense 32-bit limbs (exact NCCL int64 sum)
//   k_agg_import     summed limbs -> aggregate relation (groups with rows, ascending code)
#include <cuda_runtime.h>
#include <stdint.h>

#include "dist_kernels.h"
#include "internal.h"

namespace rw {

// ---------------------------------------------------------------------------
// column access with the declared type (lexicographic comparison in each type)
// ---------------------------------------------------------------------------
__device__ __forceinline__ int cmp_val(const void *c, int type, int64_t i, const void *d, int64_t j)
{
    switch (type) {
    case T_I32: { int32_t a = ((const int32_t *)c)[i], b = ((const int32_t *)d)[j]; return (a > b) - (a < b); }
    case T_U32: { uint32_t a = ((const uint32_t *)c)[i], b = ((const uint32_t *)d)[j]; return (a > b) - (a < b); }
    case T_I64: { int64_t a = ((const int64_t *)c)[i], b = ((const int64_t *)d)[j]; return (a > b) - (a < b); }
    case T_U64: { uint64_t a = ((const uint64_t *)c)[i], b = ((const uint64_t *)d)[j]; return (a > b) - (a < b); }
    default: { uint8_t a = ((const uint8_t *)c)[i], b = ((const uint8_t *)d)[j]; return (a > b) - (a < b); }
    }
}

// a[i] <= b[j] over all columns
__device__ __forceinline__ bool tuple_le(const MergeCols &A, int64_t i, const MergeCols &B, int64_t j, int ncols,
                                         const uint8_t *types)
{
    for (int c = 0; c < ncols; c++) {
        int r = cmp_val(A.col[c], types[c], i, B.col[c], j);
        if (r != 0)
            return r < 0;
    }
    return true;
}

__device__ __forceinline__ void copy_row(const MergeCols &S, int64_t i, MergeOut &D, int64_t o, int ncols,
                                         const uint8_t *types)
{
    for (int c = 0; c < ncols; c++) {
        switch (type_width(types[c])) {
        case 1: ((uint8_t *)D.col[c])[o] = ((const uint8_t *)S.col[c])[i]; break;
        case 4: ((uint32_t *)D.col[c])[o] = ((const uint32_t *)S.col[c])[i]; break;
        default: ((uint64_t *)D.col[c])[o] = ((const uint64_t *)S.col[c])[i]; break;
        }
    }
}

// lower bound of each splitter in a sorted key column (rows with key < splitter)
template <typename K>
__global__ void k_split_bounds(const K *keys, int64_t n, const K *spl, int nsplit, int64_t *bounds)
{
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= nsplit)
        return;
    const K s = spl[j];
    int64_t lo = 0, hi = n;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (keys[mid] < s) lo = mid + 1;
        else hi = mid;
    }
    bounds[j] = lo;
}

// Merge path over (A, B): each thread owns kMergeItems consecutive outputs, finds its
// split with a diagonal binary search, then merges sequentially.  Ties take A first,
// so merging per-rank runs in rank order is stable.
constexpr int kMergeItems = 8;

__global__ void __launch_bounds__(256) k_merge2(MergeCols A, int64_t na, MergeCols B, int64_t nb, MergeOut O,
                                                int ncols, MergeTypes T)
{
    const int64_t total = na + nb;
    const int64_t d = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * kMergeItems;
    if (d >= total)
        return;
    int64_t lo = d > nb ? d - nb : 0, hi = d < na ? d : na;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        // A[mid] goes before B[d - mid - 1] iff A[mid] <= B[d - mid - 1]
        if (tuple_le(A, mid, B, d - mid - 1, ncols, T.t))
            lo = mid + 1;
        else
            hi = mid;
    }
    int64_t i = lo, j = d - lo;
    const int64_t end = d + kMergeItems < total ? d + kMergeItems : total;
    for (int64_t o = d; o < end; o++) {
        const bool take_a = j >= nb || (i < na && tuple_le(A, i, B, j, ncols, T.t));
        if (take_a)
            copy_row(A, i++, O, o, ncols, T.t);
        else
            copy_row(B, j++, O, o, ncols, T.t);
    }
}

// ---------------------------------------------------------------------------
// aggregate limbs
// ---------------------------------------------------------------------------
__global__ void k_agg_export(AggXfer X, const int64_t *n_dev, int64_t n_host, int64_t *limbs)
{
    const int64_t n = n_dev ? *n_dev : n_host;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t g = 0;
        for (int c = 0; c < X.ngc; c++) {
            uint64_t code;
            switch (type_width(X.gtype[c])) {
            case 1: code = ((const uint8_t *)X.col[c])[i]; break;
            case 4: code = ((const uint32_t *)X.col[c])[i]; break;
            default: code = ((const uint64_t *)X.col[c])[i]; break;
            }
            g = g * X.gdomain[c] + (int64_t)code;
        }
        int64_t *L = limbs + g * X.L;
        L[0] = 1;                                  // group present on this rank
        int oc = X.ngc, lc = 1;
        for (int q = 0; q < X.nreq; q++) {
            if (X.is_sum[q]) {
                const uint64_t lo = ((const uint64_t *)X.col[oc])[i];
                const uint64_t hv = ((const uint64_t *)X.col[oc + 1])[i];
                L[lc + 0] = (int64_t)(lo & 0xffffffffull);
                L[lc + 1] = (int64_t)(lo >> 32);
                L[lc + 2] = (int64_t)(hv & 0xffffffffull);
                L[lc + 3] = (int64_t)(hv >> 32);
                oc += 2;
                lc += 4;
            } else {
                L[lc] = ((const int64_t *)X.col[oc])[i];
                oc += 1;
                lc += 1;
            }
        }
    }
}

__global__ void __launch_bounds__(256) k_agg_import(AggXfer X, const int64_t *limbs, OutPtrs out, int64_t cap,
                                                    int64_t *n_dev)
{
    __shared__ uint32_t wsum[8];
    __shared__ int64_t base;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0)
        base = 0;
    __syncthreads();
    for (int g0 = 0; g0 < X.D; g0 += 256) {
        const int g = g0 + tid;
        const bool live = g < X.D && limbs[(int64_t)g * X.L] > 0;
        const uint32_t b = __ballot_sync(0xffffffffu, live);
        if (lane == 0)
            wsum[warp] = __popc(b);
        __syncthreads();
        uint32_t before = 0, total = 0;
        for (int w = 0; w < 8; w++) {
            if (w < warp) before += wsum[w];
            total += wsum[w];
        }
        uint32_t lt;
        asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
        const int64_t pos = base + before + __popc(b & lt);
        if (live && pos < cap) {
            const int64_t *L = limbs + (int64_t)g * X.L;
            int rem = g;
            int codes[kMaxGroupCols];
            for (int c = X.ngc - 1; c >= 0; c--) {
                codes[c] = rem % X.gdomain[c];
                rem /= X.gdomain[c];
            }
            int oc = 0;
            for (int c = 0; c < X.ngc; c++, oc++) {
                switch (type_width(X.gtype[c])) {
                case 1: ((uint8_t *)out.col[oc])[pos] = (uint8_t)codes[c]; break;
                case 4: ((uint32_t *)out.col[oc])[pos] = (uint32_t)codes[c]; break;
                default: ((uint64_t *)out.col[oc])[pos] = (uint64_t)codes[c]; break;
                }
            }
            int lc = 1;
            for (int q = 0; q < X.nreq; q++) {
                if (X.is_sum[q]) {
                    // value = sum_k limb_k * 2^(32k) mod 2^128 (limb sums are exact in int64)
                    unsigned __int128 v = 0;
                    for (int k = 3; k >= 0; k--)
                        v = (v << 32) + (unsigned __int128)(uint64_t)L[lc + k];
                    ((uint64_t *)out.col[oc])[pos] = (uint64_t)v;
                    ((uint64_t *)out.col[oc + 1])[pos] = (uint64_t)(v >> 64);
                    oc += 2;
                    lc += 4;
                } else {
                    ((int64_t *)out.col[oc])[pos] = L[lc];
                    oc += 1;
                    lc += 1;
                }
            }
        }
        __syncthreads();
        if (tid == 0)
            base += total;
        __syncthreads();
    }
    if (tid == 0)
        *n_dev = base;
}

// ---------------------------------------------------------------------------
// launchers
// ---------------------------------------------------------------------------
cudaError_t split_bounds_launch(const void *keys, int64_t n, int key_type, const void *spl, int nsplit,
                                int64_t *bounds, cudaStream_t s)
{
    if (nsplit <= 0)
        return cudaSuccess;
    const int grid = (nsplit + 127) / 128;
    switch (key_type) {
    case T_I32: k_split_bounds<int32_t><<<grid, 128, 0, s>>>((const int32_t *)keys, n, (const int32_t *)spl, nsplit, bounds); break;
    case T_U32: k_split_bounds<uint32_t><<<grid, 128, 0, s>>>((const uint32_t *)keys, n, (const uint32_t *)spl, nsplit, bounds); break;
    case T_I64: k_split_bounds<int64_t><<<grid, 128, 0, s>>>((const int64_t *)keys, n, (const int64_t *)spl, nsplit, bounds); break;
    case T_U64: k_split_bounds<uint64_t><<<grid, 128, 0, s>>>((const uint64_t *)keys, n, (const uint64_t *)spl, nsplit, bounds); break;
    default: k_split_bounds<uint8_t><<<grid, 128, 0, s>>>((const uint8_t *)keys, n, (const uint8_t *)spl, nsplit, bounds); break;
    }
    return cudaGetLastError();
}

cudaError_t merge2_launch(const MergeCols &A, int64_t na, const MergeCols &B, int64_t nb, const MergeOut &O,
                          int ncols, const MergeTypes &T, cudaStream_t s)
{
    const int64_t threads = (na + nb + kMergeItems - 1) / kMergeItems;
    if (threads == 0)
        return cudaSuccess;
    k_merge2<<<(unsigned)((threads + 255) / 256), 256, 0, s>>>(A, na, B, nb, O, ncols, T);
    return cudaGetLastError();
}

cudaError_t agg_export_launch(const AggXfer &X, const int64_t *n_dev, int64_t n_host, int64_t *limbs, cudaStream_t s)
{
    k_agg_export<<<4, 256, 0, s>>>(X, n_dev, n_host, limbs);
    return cudaGetLastError();
}

cudaError_t agg_import_launch(const AggXfer &X, const int64_t *limbs, const OutPtrs &out, int64_t cap,
                              int64_t *n_dev, cudaStream_t s)
{
    k_agg_import<<<1, 256, 0, s>>>(X, limbs, out, cap, n_dev);
    return cudaGetLastError();
}

}  // namespace rw
