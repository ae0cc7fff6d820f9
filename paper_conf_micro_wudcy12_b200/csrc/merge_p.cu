// merge_p.cu — single-pass P-way merge of the runs a key-range exchange receives
// ("all-to-all over NVLink, then a merge of the P received runs";
// P:196 §4.3.2 merge-path partitioning, generalised from two inputs to P).
//
// Every run is sorted on the whole tuple; the merged order is the total order
// (tuple, run, position), so equal tuples keep run (= rank) order.  Tuples of <= 8
// bytes are handled as one order-preserving u64 image (columns concatenated, first
// column most significant, signed types with the sign bit flipped).
//
//   k_mp_samples  every T-th element of every run becomes a sample; its u64 image
//                 is stored (S samples, a sparse index of each run, L2-resident)
//   k_mp_cuts     for every (sample s, run q): cut_q(s) = the number of run-q
//                 elements before s in the total order -- a binary search over run
//                 q's samples, then inside one T-element window of run q
//   k_mp_bounds   a sample's rank among all samples is j + sum_q ceil(cut_q / T);
//                 every G-th sample (in that order) starts a merge group
//   k_mp_merge    one CTA per group: the group's P segments [cut(start), cut(end))
//                 hold at most (G + P) * T = kMpC elements; they are read once
//                 (coalesced per column), merged in shared memory by ceil(log2 P)
//                 pairwise merge-path rounds, and written once at offset
//                 sum_q cut_q(start) -- one HBM read and one write of the data,
//                 against ceil(log2 P) read+write passes of a pairwise merge tree.
#include <cuda_runtime.h>
#include <stdint.h>

#include "dist_kernels.h"
#include "internal.h"

namespace rw {

// order-preserving image of one value (signed: sign bit flipped), width-masked
__device__ __forceinline__ uint64_t mp_okey(const void *col, int type, int64_t i)
{
    switch (type) {
    case T_I32: return (uint64_t)(((const uint32_t *)col)[i] ^ 0x80000000u);
    case T_U32: return (uint64_t)((const uint32_t *)col)[i];
    case T_I64: return ((const uint64_t *)col)[i] ^ 0x8000000000000000ull;
    case T_U64: return ((const uint64_t *)col)[i];
    default: return (uint64_t)((const uint8_t *)col)[i];
    }
}

__device__ __forceinline__ uint64_t mp_pack(const void *const *col, const uint8_t *types, int ncols, int64_t i)
{
    uint64_t k = 0;
    for (int c = 0; c < ncols; c++) {
        const int w = type_width(types[c]);
        const uint64_t v = mp_okey(col[c], types[c], i);
        k = w == 8 ? v : ((k << (8 * w)) | v);
    }
    return k;
}

__device__ __forceinline__ void mp_unpack(void *const *out, const uint8_t *types, int ncols, int64_t o, uint64_t k)
{
    for (int c = ncols - 1; c >= 0; c--) {
        const int w = type_width(types[c]);
        const uint64_t v = w == 8 ? k : (k & ((1ull << (8 * w)) - 1));
        switch (types[c]) {
        case T_I32: ((uint32_t *)out[c])[o] = (uint32_t)v ^ 0x80000000u; break;
        case T_U32: ((uint32_t *)out[c])[o] = (uint32_t)v; break;
        case T_I64: ((uint64_t *)out[c])[o] = v ^ 0x8000000000000000ull; break;
        case T_U64: ((uint64_t *)out[c])[o] = v; break;
        default: ((uint8_t *)out[c])[o] = (uint8_t)v; break;
        }
        k = w == 8 ? 0 : (k >> (8 * w));
    }
}

// element i of run q as its u64 image
__device__ __forceinline__ uint64_t mp_load(const MpLaunch &M, int q, int64_t i)
{
    const int64_t r = M.run_off[q] + i;
    return M.packed ? M.packed[r] : mp_pack(M.col, M.types, M.ncols, r);
}

__device__ __forceinline__ int mp_run_of_sample(const MpLaunch &M, int64_t s)
{
    int p = 0;
    while (p + 1 < M.nrun && M.samp_base[p + 1] <= s)
        p++;
    return p;
}

__global__ void k_mp_samples(const __grid_constant__ MpLaunch M)
{
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < M.S; s += (int64_t)gridDim.x * blockDim.x) {
        const int p = mp_run_of_sample(M, s);
        M.sv[s] = mp_load(M, p, (s - M.samp_base[p]) * M.T);
    }
}

// cut_q(s): run-q elements before sample s = (p, j) in the order (tuple, run, position):
// q < p counts elements <= v, q > p counts elements < v, q == p is the position j*T.
__global__ void k_mp_cuts(const __grid_constant__ MpLaunch M)
{
    const int64_t total = M.S * M.nrun;
    for (int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; x < total; x += (int64_t)gridDim.x * blockDim.x) {
        const int64_t s = x / M.nrun;
        const int q = (int)(x - s * M.nrun);
        const int p = mp_run_of_sample(M, s);
        int64_t cut;
        if (q == p) {
            cut = (s - M.samp_base[p]) * M.T;
        } else {
            const uint64_t v = M.sv[s];
            const bool le = q < p;
            // stage 1: how many of run q's samples precede s
            int64_t lo = M.samp_base[q], hi = M.samp_base[q + 1];
            const int64_t first = lo;
            while (lo < hi) {
                const int64_t mid = (lo + hi) >> 1;
                const uint64_t w = M.sv[mid];
                if (le ? w <= v : w < v) lo = mid + 1;
                else hi = mid;
            }
            const int64_t c1 = lo - first;
            if (c1 == 0) {
                cut = 0;
            } else {
                // stage 2: inside the window (jT, min((j+1)T, n_q)] of run q
                const int64_t nq = M.run_off[q + 1] - M.run_off[q];
                int64_t a = (c1 - 1) * M.T + 1, b = c1 * M.T < nq ? c1 * M.T : nq;
                while (a < b) {
                    const int64_t mid = (a + b) >> 1;
                    const uint64_t w = mp_load(M, q, mid);
                    if (le ? w <= v : w < v) a = mid + 1;
                    else b = mid;
                }
                cut = a;
            }
        }
        M.cuts[x] = (uint32_t)cut;
    }
}

__global__ void k_mp_bounds(const __grid_constant__ MpLaunch M)
{
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < M.S; s += (int64_t)gridDim.x * blockDim.x) {
        const int p = mp_run_of_sample(M, s);
        int64_t R = s - M.samp_base[p];
        for (int q = 0; q < M.nrun; q++)
            if (q != p)
                R += ((int64_t)M.cuts[s * M.nrun + q] + M.T - 1) / M.T;
        if (R % M.G == 0)
            M.bound[R / M.G] = s;
    }
}

__global__ void __launch_bounds__(kMpThreads, 3) k_mp_merge(const __grid_constant__ MpLaunch M)
{
    extern __shared__ __align__(16) uint64_t mp_smem[];
    uint64_t *bufA = mp_smem, *bufB = mp_smem + kMpC;
    __shared__ int32_t st[kMpMaxRuns + 1], st2[kMpMaxRuns + 1];
    __shared__ int64_t c0[kMpMaxRuns];
    __shared__ int64_t obase;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    constexpr int NW = kMpThreads / 32;
    for (int64_t g = blockIdx.x; g < M.NG; g += gridDim.x) {
        if (tid < 32) {
            const int q = lane;
            int32_t len = 0;
            int64_t c = 0;
            if (q < M.nrun) {
                c = M.cuts[M.bound[g] * M.nrun + q];
                const int64_t e = g + 1 < M.NG ? (int64_t)M.cuts[M.bound[g + 1] * M.nrun + q]
                                               : M.run_off[q + 1] - M.run_off[q];
                len = (int32_t)(e - c);
                c0[q] = c;
            }
            // inclusive scans of the segment lengths and the start cuts
            int32_t inc = len;
            int64_t cs = c;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int32_t y = __shfl_up_sync(0xffffffffu, inc, o);
                const int64_t z = __shfl_up_sync(0xffffffffu, cs, o);
                if (lane >= o) {
                    inc += y;
                    cs += z;
                }
            }
            if (q < M.nrun)
                st[q + 1] = inc;
            if (q == 0)
                st[0] = 0;
            if (q == M.nrun - 1)
                obase = cs;
        }
        __syncthreads();
        const int m = st[M.nrun];
        if (m > kMpC)
            __trap();   // cannot happen: a group holds at most (G + P) * T <= kMpC elements
        // read the segments once, coalesced per column, as u64 images
        for (int q = warp; q < M.nrun; q += NW) {
            const int a = st[q], len = st[q + 1] - a;
            for (int t = lane; t < len; t += 32)
                bufA[a + t] = mp_load(M, q, c0[q] + t);
        }
        __syncthreads();
        // pairwise merge-path rounds over adjacent segments (left first on ties)
        int nseg = M.nrun;
        uint64_t *src = bufA, *dst = bufB;
        while (nseg > 1) {
            const int npair = (nseg + 1) >> 1;
            const int d0 = tid * kMpItems;
            const int end = d0 + kMpItems < m ? d0 + kMpItems : m;
            int o = d0;
            int k = 0;
            while (o < end) {
                while (k + 1 < npair && st[2 * (k + 1)] <= o)
                    k++;
                const int a0 = st[2 * k];
                const int a1 = st[2 * k + 1 < nseg ? 2 * k + 1 : nseg];
                const int b1 = st[2 * k + 2 < nseg ? 2 * k + 2 : nseg];
                const int na = a1 - a0, nb = b1 - a1, diag = o - a0;
                int lo = diag > nb ? diag - nb : 0, hi = diag < na ? diag : na;
                while (lo < hi) {
                    const int mid = (lo + hi) >> 1;
                    if (src[a0 + mid] <= src[a1 + diag - mid - 1]) lo = mid + 1;
                    else hi = mid;
                }
                int i = lo, j = diag - lo;
                const int stop = end < b1 ? end : b1;
                uint64_t x = i < na ? src[a0 + i] : 0, y = j < nb ? src[a1 + j] : 0;
                for (; o < stop; o++) {
                    const bool take_a = j >= nb || (i < na && x <= y);
                    if (take_a) {
                        dst[o] = x;
                        i++;
                        x = i < na ? src[a0 + i] : 0;
                    } else {
                        dst[o] = y;
                        j++;
                        y = j < nb ? src[a1 + j] : 0;
                    }
                }
            }
            __syncthreads();
            if (tid <= npair)
                st2[tid] = tid < npair ? st[2 * tid] : m;
            __syncthreads();
            if (tid <= npair)
                st[tid] = st2[tid];
            nseg = npair;
            uint64_t *t = src;
            src = dst;
            dst = t;
            __syncthreads();
        }
        // write once, coalesced per column
        const int64_t ob = obase;
        for (int t = tid; t < m; t += kMpThreads)
            mp_unpack(M.out, M.types, M.ncols, ob + t, src[t]);
        __syncthreads();
    }
}

__global__ void k_mp_pack(const __grid_constant__ MpLaunch M, int64_t n, uint64_t *dst)
{
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] = mp_pack(M.col, M.types, M.ncols, i);
}

cudaError_t mp_pack_launch(const MpLaunch &M, int64_t n, uint64_t *dst, int sms, cudaStream_t s)
{
    if (n <= 0)
        return cudaSuccess;
    const int64_t want = (n + 255) / 256;
    const int grid = (int)(want < (int64_t)sms * 8 ? want : (int64_t)sms * 8);
    k_mp_pack<<<grid, 256, 0, s>>>(M, n, dst);
    return cudaGetLastError();
}

cudaError_t mp_merge_launch(const MpLaunch &M, int sms, cudaStream_t s)
{
    auto grid_for = [&](int64_t work) {
        const int64_t want = (work + 255) / 256;
        return (int)(want < (int64_t)sms * 16 ? (want > 0 ? want : 1) : (int64_t)sms * 16);
    };
    k_mp_samples<<<grid_for(M.S), 256, 0, s>>>(M);
    k_mp_cuts<<<grid_for(M.S * M.nrun), 256, 0, s>>>(M);
    k_mp_bounds<<<grid_for(M.S), 256, 0, s>>>(M);
    static bool attr = false;
    const int smem = 2 * kMpC * (int)sizeof(uint64_t);
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_mp_merge, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess)
            return e;
        attr = true;
    }
    const int64_t grid = M.NG < (int64_t)sms * 3 ? M.NG : (int64_t)sms * 3;
    k_mp_merge<<<(unsigned)grid, kMpThreads, smem, s>>>(M);
    return cudaGetLastError();
}

}  // namespace rw
