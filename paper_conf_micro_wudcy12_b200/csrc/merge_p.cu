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
//   k_mp_rank     a sample's rank among all samples = j + the samples of the other
//                 runs before it (binary searches over the L2-resident sample images);
//                 every G-th sample in that order starts a merge group
//   k_mp_cuts     for every (group start s, run q): cut_q(s) = the number of run-q
//                 elements before s in the total order -- the samples locate one
//                 T-element window of run q, a binary search inside it the cut
//   k_mp_merge    one CTA per group: the group's P segments [cut(start), cut(end))
//                 hold at most (G + P) * T = kMpC elements; they are read once
//                 (coalesced per column), merged in shared memory (padded against bank
//                 conflicts) by ceil(log2 P)
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

// Number of run-q samples before value v in the order (tuple, run, position) of a
// sample of run p: q < p counts samples <= v, q > p counts samples < v.
__device__ __forceinline__ int64_t mp_samples_before(const MpLaunch &M, int q, int p, uint64_t v)
{
    const bool le = q < p;
    int64_t lo = M.samp_base[q], hi = M.samp_base[q + 1];
    const int64_t first = lo;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        const uint64_t w = M.sv[mid];
        if (le ? w <= v : w < v) lo = mid + 1;
        else hi = mid;
    }
    return lo - first;
}

// A sample's rank among all samples: j + sum_{q != p} (run-q samples before it).  The
// samples of rank 0, G, 2G, ... start the merge groups.  Only the L2-resident sample
// images are read (no data).
__global__ void k_mp_rank(const __grid_constant__ MpLaunch M)
{
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < M.S; s += (int64_t)gridDim.x * blockDim.x) {
        const int p = mp_run_of_sample(M, s);
        const uint64_t v = M.sv[s];
        int64_t R = s - M.samp_base[p];
        for (int q = 0; q < M.nrun; q++)
            if (q != p)
                R += mp_samples_before(M, q, p, v);
        if (R % M.G == 0)
            M.bound[R / M.G] = s;
    }
}

// cut_q(g): run-q elements before group g's start sample s = (p, j) in the order
// (tuple, run, position): q < p counts elements <= v, q > p counts elements < v,
// q == p is the position j*T -- the samples locate a T-element window of run q, a
// binary search inside it finds the cut.
__global__ void k_mp_cuts(const __grid_constant__ MpLaunch M)
{
    const int64_t total = M.NG * M.nrun;
    for (int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; x < total; x += (int64_t)gridDim.x * blockDim.x) {
        const int64_t g = x / M.nrun;
        const int q = (int)(x - g * M.nrun);
        const int64_t s = M.bound[g];
        const int p = mp_run_of_sample(M, s);
        int64_t cut;
        if (q == p) {
            cut = (s - M.samp_base[p]) * M.T;
        } else {
            const uint64_t v = M.sv[s];
            const bool le = q < p;
            const int64_t c1 = mp_samples_before(M, q, p, v);
            if (c1 == 0) {
                cut = 0;
            } else {
                // inside the window (jT, min((j+1)T, n_q)] of run q
                const int64_t nq = M.run_off[q + 1] - M.run_off[q];
                int64_t lo = (c1 - 1) * M.T + 1, hi = c1 * M.T < nq ? c1 * M.T : nq;
                while (lo < hi) {
                    const int64_t mid = (lo + hi) >> 1;
                    const uint64_t w = mp_load(M, q, mid);
                    if (le ? w <= v : w < v) lo = mid + 1;
                    else hi = mid;
                }
                cut = lo;
            }
        }
        M.cuts[x] = (uint32_t)cut;
    }
}

// shared-memory index with one pad word per 16: the merge walks of neighbouring lanes
// (8 or 16 elements apart) fall into different banks
__device__ __forceinline__ int mp_pi(int i) { return i + (i >> 4); }

__global__ void __launch_bounds__(kMpThreads, 3) k_mp_merge(const __grid_constant__ MpLaunch M)
{
    extern __shared__ __align__(16) uint64_t mp_smem[];
    uint64_t *bufA = mp_smem, *bufB = mp_smem + kMpCP;
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
                c = M.cuts[g * M.nrun + q];
                const int64_t e = g + 1 < M.NG ? (int64_t)M.cuts[(g + 1) * M.nrun + q]
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
            const int64_t c = M.run_off[q] + c0[q];
            if (M.packed) {
                int t = lane;
                for (; t + 96 < len; t += 128) {
                    uint64_t v[4];
#pragma unroll
                    for (int u = 0; u < 4; u++)
                        v[u] = M.packed[c + t + 32 * u];
#pragma unroll
                    for (int u = 0; u < 4; u++)
                        bufA[mp_pi(a + t + 32 * u)] = v[u];
                }
                for (; t < len; t += 32)
                    bufA[mp_pi(a + t)] = M.packed[c + t];
            } else {
                // column by column (type dispatch outside the row loop, independent loads
                // in flight), each column's image shifted into the staged u64 words
                for (int cc = 0; cc < M.ncols; cc++) {
                    const int ty = M.types[cc];
                    const int w = type_width(ty);
                    const uint64_t flip = ty == T_I32 ? 0x80000000ull : ty == T_I64 ? 0x8000000000000000ull : 0ull;
                    for (int t0 = lane; t0 < len; t0 += 128) {
                        uint64_t v[4];
#pragma unroll
                        for (int u = 0; u < 4; u++) {
                            const int t = t0 + 32 * u;
                            v[u] = 0;
                            if (t < len) {
                                if (w == 4) v[u] = (uint64_t)((const uint32_t *)M.col[cc])[c + t];
                                else if (w == 8) v[u] = ((const uint64_t *)M.col[cc])[c + t];
                                else v[u] = (uint64_t)((const uint8_t *)M.col[cc])[c + t];
                            }
                        }
#pragma unroll
                        for (int u = 0; u < 4; u++) {
                            const int t = t0 + 32 * u;
                            if (t < len) {
                                uint64_t &d = bufA[mp_pi(a + t)];
                                d = (w == 8 || cc == 0) ? (v[u] ^ flip) : ((d << (8 * w)) | (v[u] ^ flip));
                            }
                        }
                    }
                }
            }
        }
        __syncthreads();
        // pairwise merge-path rounds over adjacent segments (left first on ties); the
        // segment starts alternate between st and st2 (one barrier per round)
        int nseg = M.nrun;
        uint64_t *src = bufA, *dst = bufB;
        int32_t *cs = st, *ns = st2;
        while (nseg > 1) {
            const int npair = (nseg + 1) >> 1;
            const int d0 = tid * kMpItems;
            const int end = d0 + kMpItems < m ? d0 + kMpItems : m;
            int o = d0;
            int k = 0;
            while (o < end) {
                while (k + 1 < npair && cs[2 * (k + 1)] <= o)
                    k++;
                const int a0 = cs[2 * k];
                const int a1 = cs[2 * k + 1 < nseg ? 2 * k + 1 : nseg];
                const int b1 = cs[2 * k + 2 < nseg ? 2 * k + 2 : nseg];
                const int na = a1 - a0, nb = b1 - a1, diag = o - a0;
                int lo = diag > nb ? diag - nb : 0, hi = diag < na ? diag : na;
                while (lo < hi) {
                    const int mid = (lo + hi) >> 1;
                    if (src[mp_pi(a0 + mid)] <= src[mp_pi(a1 + diag - mid - 1)]) lo = mid + 1;
                    else hi = mid;
                }
                // branch-free walk: one shared load per output (the taken side's next)
                int ia = a0 + lo, jb = a1 + diag - lo;
                const int stop = end < b1 ? end : b1;
                uint64_t x = ia < a1 ? src[mp_pi(ia)] : 0, y = jb < b1 ? src[mp_pi(jb)] : 0;
                for (; o < stop; o++) {
                    const bool ta = jb >= b1 || (ia < a1 && x <= y);
                    dst[mp_pi(o)] = ta ? x : y;
                    const int nx = ta ? ia + 1 : jb + 1;
                    const uint64_t v = nx < (ta ? a1 : b1) ? src[mp_pi(nx)] : 0;
                    ia = ta ? nx : ia;
                    jb = ta ? jb : nx;
                    x = ta ? v : x;
                    y = ta ? y : v;
                }
            }
            if (tid <= npair)
                ns[tid] = tid < npair ? cs[2 * tid] : m;
            __syncthreads();
            nseg = npair;
            uint64_t *t = src;
            src = dst;
            dst = t;
            int32_t *u = cs;
            cs = ns;
            ns = u;
        }
        // write once, coalesced per column (common layouts without the type dispatch)
        const int64_t ob = obase;
        if (M.ncols == 2 && type_width(M.types[0]) == 4 && type_width(M.types[1]) == 4) {
            const uint32_t f0 = M.types[0] == T_I32 ? 0x80000000u : 0u, f1 = M.types[1] == T_I32 ? 0x80000000u : 0u;
            uint32_t *o0 = (uint32_t *)M.out[0] + ob, *o1 = (uint32_t *)M.out[1] + ob;
            for (int t = tid; t < m; t += kMpThreads) {
                const uint64_t v = src[mp_pi(t)];
                o0[t] = (uint32_t)(v >> 32) ^ f0;
                o1[t] = (uint32_t)v ^ f1;
            }
        } else if (M.ncols == 1 && type_width(M.types[0]) == 8) {
            const uint64_t f = M.types[0] == T_I64 ? 0x8000000000000000ull : 0ull;
            uint64_t *o0 = (uint64_t *)M.out[0] + ob;
            for (int t = tid; t < m; t += kMpThreads)
                o0[t] = src[mp_pi(t)] ^ f;
        } else {
            for (int t = tid; t < m; t += kMpThreads)
                mp_unpack(M.out, M.types, M.ncols, ob + t, src[mp_pi(t)]);
        }
        __syncthreads();
    }
}

__global__ void k_mp_pack(const __grid_constant__ MpLaunch M, int64_t n, uint64_t *dst)
{
    // 4 consecutive tuples per thread: independent loads in flight, two 16-byte stores
    const int64_t n4 = n / 4;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
        uint64_t v[4];
#pragma unroll
        for (int u = 0; u < 4; u++)
            v[u] = mp_pack(M.col, M.types, M.ncols, 4 * i + u);
        ((ulonglong2 *)dst)[2 * i] = make_ulonglong2(v[0], v[1]);
        ((ulonglong2 *)dst)[2 * i + 1] = make_ulonglong2(v[2], v[3]);
    }
    for (int64_t i = 4 * n4 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
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
    k_mp_rank<<<grid_for(M.S), 256, 0, s>>>(M);
    k_mp_cuts<<<grid_for(M.NG * M.nrun), 256, 0, s>>>(M);
    static bool attr = false;
    const int smem = 2 * kMpCP * (int)sizeof(uint64_t);
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
