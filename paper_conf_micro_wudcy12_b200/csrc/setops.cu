// setops.cu — SET UNION / SET INTERSECTION / SET DIFFERENCE (Table 1,
// reading A24: whole-tuple membership, set semantics, inputs sorted on every
// attribute, ascending output) on the merge-path machinery of the JOIN
// (§4.3.3 sizes the INTERSECT output by min(|x|, |y|)).
//
// The merged order of x and y (x first on equal tuples, P:196 binary-search
// partitioning) puts every distinct tuple value into one contiguous segment
// [its x rows][its y rows].  With pred / succ the merged neighbours of an element e:
//   UNION      emits e  iff  pred != e                      (first row of each segment)
//   INTERSECT  emits e  iff  e in y, pred in x, pred == e    (the x->y step of a segment)
//   DIFFERENCE emits e  iff  e in x, succ != e               (last x row of a segment
//                                                            that has no y row)
// so each segment emits at most once and the output is ascending without a sort.
//   k_set_splits   merge-path split of every partition boundary (2048 merged rows)
//                  and the boundary's merged neighbours;
//   k_set_op       per partition: stage both inputs' rows in smem as order-preserving
//                  u64 keys (one packed key when a tuple is <= 8 bytes), merge walk
//                  (8 positions per thread), emission flags, block scan, decoupled
//                  look-back over the partitions for the output offset, store.
// (diagnostics: a count pass + k_set_scan + a write pass instead of the look-back)
#include "chain.cuh"
#include "kernels.h"

namespace rw {

constexpr int kSetItems = 8;
constexpr int kSetT = kThreads * kSetItems;     // merged rows per partition

// order-preserving 64-bit image of a value (signed types: sign bit flipped)
__device__ __forceinline__ uint64_t okey(const void *col, int type, int64_t i)
{
    switch (type) {
    case T_I32: return (uint64_t)(((const uint32_t *)col)[i] ^ 0x80000000u);
    case T_U32: return ((const uint32_t *)col)[i];
    case T_I64: return ((const uint64_t *)col)[i] ^ 0x8000000000000000ull;
    case T_U64: return ((const uint64_t *)col)[i];
    default: return ((const uint8_t *)col)[i];
    }
}

__device__ __forceinline__ void store_okey(void *col, int type, int64_t i, uint64_t k)
{
    switch (type) {
    case T_I32: ((uint32_t *)col)[i] = (uint32_t)k ^ 0x80000000u; break;
    case T_U32: ((uint32_t *)col)[i] = (uint32_t)k; break;
    case T_I64: ((uint64_t *)col)[i] = k ^ 0x8000000000000000ull; break;
    case T_U64: ((uint64_t *)col)[i] = k; break;
    default: ((uint8_t *)col)[i] = (uint8_t)k; break;
    }
}

// Tuples whose columns total <= 8 bytes are staged as ONE packed key: the columns'
// order-preserving images concatenated, first column most significant, so a tuple
// compare is a single u64 compare (e.g. (u32 key, u32 val) -> key << 32 | val).
__device__ __forceinline__ uint64_t pack_row(const SetLaunch &S, const void *const *a, int64_t i)
{
    uint64_t k = 0;
    for (int c = 0; c < S.ncols; c++) {
        const int w = type_width(S.types[c]);
        const uint64_t v = okey(a[c], S.types[c], i);
        const uint64_t img = w == 4 ? (uint64_t)(uint32_t)v : w == 1 ? (v & 0xffu) : v;
        k = w == 8 ? img : ((k << (8 * w)) | img);
    }
    return k;
}

__device__ __forceinline__ void store_packed(const SetLaunch &S, int64_t o, uint64_t k)
{
    for (int c = S.ncols - 1; c >= 0; c--) {
        const int w = type_width(S.types[c]);
        const uint64_t v = w == 8 ? k : (k & ((1ull << (8 * w)) - 1));
        store_okey(S.out[c], S.types[c], o, S.types[c] == T_I32 ? (v & 0xffffffffull) : v);
        k = w == 8 ? 0 : (k >> (8 * w));
    }
}

// lexicographic compare of global rows x[i] and y[j]: <0, 0, >0
__device__ inline int gcmp(const SetLaunch &S, const void *const *a, int64_t i, const void *const *b, int64_t j)
{
    for (int c = 0; c < S.ncols; c++) {
        const uint64_t u = okey(a[c], S.types[c], i), v = okey(b[c], S.types[c], j);
        if (u != v)
            return u < v ? -1 : 1;
    }
    return 0;
}

// smem rows: column c of staged row r at s[c * kSetS + r]
constexpr int kSetS = kSetT + 2;                // + pred and succ slots
template <int NC>
__device__ __forceinline__ int scmp(const uint64_t *s, int r, int q)
{
#pragma unroll
    for (int c = 0; c < NC; c++) {
        const uint64_t u = s[c * kSetS + r], v = s[c * kSetS + q];
        if (u != v)
            return u < v ? -1 : 1;
    }
    return 0;
}

__global__ void k_set_splits(const __grid_constant__ SetLaunch S)
{
    const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (p > S.nparts)
        return;
    const int64_t d = min(p * kSetT, S.nx + S.ny);
    int64_t lo = d > S.ny ? d - S.ny : 0, hi = d < S.nx ? d : S.nx;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (gcmp(S, S.x, mid, S.y, d - mid - 1) <= 0)   // x first on equal tuples
            lo = mid + 1;
        else
            hi = mid;
    }
    S.split[p] = lo;
    // merged neighbours of the boundary: pred = element d-1 (the later of x[lo-1],
    // y[d-lo-1]; y after x on ties), succ = element d (the earlier of x[lo], y[d-lo])
    const int64_t j = d - lo;
    const bool px = lo > 0, py = j > 0, sx = lo < S.nx, sy = j < S.ny;
    const bool pis_x = px && (!py || gcmp(S, S.x, lo - 1, S.y, j - 1) > 0);
    const bool sis_x = sx && (!sy || gcmp(S, S.x, lo, S.y, j) <= 0);
    S.nbr[p] = (int32_t)((px || py) | (pis_x << 1) | ((sx || sy) << 2) | (sis_x << 3));
}

template <int NC, bool WRITE, bool PACKED>
__global__ void __launch_bounds__(kThreads) k_set_op(const __grid_constant__ SetLaunch S)
{
    extern __shared__ __align__(16) uint64_t sm[];
    uint64_t *s = sm;                                     // ncols * kSetS staged keys
    int32_t *msrc = (int32_t *)(s + (size_t)NC * kSetS);       // merged position -> staged row
    __shared__ int32_t wcnt[kThreads / 32 + 1];
    __shared__ int32_t nbr[4];                            // has_pred, pred_is_x, has_succ, succ_is_x
    __shared__ int64_t pbase;                             // single pass: the partition's output offset
    __shared__ int64_t pclaim;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    constexpr int nc = NC;
    // single pass (look-back): partitions are claimed in order with a global atomic, so
    // every partition a CTA waits for has been claimed by a running CTA (no assumption
    // that the whole grid is resident); the count pass walks them statically
    const bool claim = WRITE && S.status != nullptr;
    // (u32 | i32) x 2 tuples with 16-byte aligned columns take the vector staging
    const bool two4 = PACKED && S.ncols == 2 && type_width(S.types[0]) == 4 && type_width(S.types[1]) == 4 &&
                      (((uintptr_t)S.x[0] | (uintptr_t)S.x[1] | (uintptr_t)S.y[0] | (uintptr_t)S.y[1]) & 15) == 0;
    const uint32_t f0 = S.types[0] == T_I32 ? 0x80000000u : 0u, f1 = S.types[1] == T_I32 ? 0x80000000u : 0u;
    // rows [start, start + n) of a two-column relation into dst[0, n): the aligned span
    // is read in 16-byte vectors (a vector never crosses a 16-byte boundary, so bytes
    // read past a column's end stay inside its allocation), out-of-range lanes skipped
    auto stage_two4 = [&](const void *const *cols, int64_t start, int n, uint64_t *dst) {
        const int64_t sa = start & ~(int64_t)3;
        const int nvec = (int)((start + n - sa + 3) / 4);
        const uint4 *c0 = (const uint4 *)((const uint32_t *)cols[0] + sa);
        const uint4 *c1 = (const uint4 *)((const uint32_t *)cols[1] + sa);
        const int sh = (int)(start - sa);
        for (int v = tid; v < nvec; v += kThreads) {
            const uint4 a = c0[v], b = c1[v];
            const uint32_t av[4] = {a.x, a.y, a.z, a.w}, bv[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const int r = 4 * v + q - sh;
                if (r >= 0 && r < n)
                    dst[r] = ((uint64_t)(av[q] ^ f0) << 32) | (uint64_t)(bv[q] ^ f1);
            }
        }
    };
    for (int64_t it = 0;; ++it) {
        int64_t p = (int64_t)blockIdx.x + it * gridDim.x;
        if (claim) {
            __syncthreads();
            if (tid == 0)
                pclaim = (int64_t)atomicAdd(&S.ctrs[0], 1u);
            __syncthreads();
            p = pclaim;
        }
        if (p >= S.nparts)
            break;
        const int64_t d0 = p * kSetT, d1 = min(d0 + kSetT, S.nx + S.ny);
        const int64_t i0 = S.split[p], i1 = S.split[p + 1], j0 = d0 - i0, j1 = d1 - i1;
        const int nX = (int)(i1 - i0), nY = (int)(j1 - j0), m = (int)(d1 - d0);
        __syncthreads();
        // stage x rows at [0, nX), y rows at [nX, nX + nY), pred at kSetT, succ at kSetT + 1
        if (PACKED && two4) {
            // two 4-byte columns: 16-byte vector loads of both columns (4 tuples per
            // thread and load, all in flight), packed key = col0 image << 32 | col1 image
            stage_two4(S.x, i0, nX, s);
            stage_two4(S.y, j0, nY, s + nX);
        } else if (PACKED) {
            for (int r = tid; r < nX; r += kThreads)
                s[r] = pack_row(S, S.x, i0 + r);
            for (int r = tid; r < nY; r += kThreads)
                s[nX + r] = pack_row(S, S.y, j0 + r);
        } else {
            for (int c = 0; c < nc; c++) {
                for (int r = tid; r < nX; r += kThreads)
                    s[c * kSetS + r] = okey(S.x[c], S.types[c], i0 + r);
                for (int r = tid; r < nY; r += kThreads)
                    s[c * kSetS + nX + r] = okey(S.y[c], S.types[c], j0 + r);
            }
        }
        // merged neighbours outside the partition (decided by k_set_splits): one
        // thread per (neighbour, column) stages them
        const int32_t fp = S.nbr[p], fs = S.nbr[p + 1];
        if (tid == 0) {
            nbr[0] = fp & 1;
            nbr[1] = (fp >> 1) & 1;
            nbr[2] = (fs >> 2) & 1;
            nbr[3] = (fs >> 3) & 1;
        }
        if (PACKED) {
            if (tid == 0 && (fp & 1))
                s[kSetT] = (fp & 2) ? pack_row(S, S.x, i0 - 1) : pack_row(S, S.y, j0 - 1);
            else if (tid == 32 && (fs & 4))
                s[kSetT + 1] = (fs & 8) ? pack_row(S, S.x, i1) : pack_row(S, S.y, j1);
        } else if (tid < nc && (fp & 1)) {
            const int c = tid;
            s[c * kSetS + kSetT] = (fp & 2) ? okey(S.x[c], S.types[c], i0 - 1) : okey(S.y[c], S.types[c], j0 - 1);
        } else if (tid >= 32 && tid < 32 + nc && (fs & 4)) {
            const int c = tid - 32;
            s[c * kSetS + kSetT + 1] = (fs & 8) ? okey(S.x[c], S.types[c], i1) : okey(S.y[c], S.types[c], j1);
        }
        __syncthreads();
        // merge walk: thread positions [dt, dt + 8) of the partition's merged order
        const int dt = tid * kSetItems;
        if (dt < m) {
            int lo = dt > nY ? dt - nY : 0, hi = dt < nX ? dt : nX;
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if (scmp<NC>(s, mid, nX + dt - mid - 1) <= 0) lo = mid + 1;
                else hi = mid;
            }
            int xi = lo, yj = dt - lo;
#pragma unroll
            for (int q = 0; q < kSetItems; q++) {
                if (dt + q < m) {
                    const bool takex = yj >= nY || (xi < nX && scmp<NC>(s, xi, nX + yj) <= 0);
                    msrc[dt + q] = takex ? xi : nX + yj;
                    xi += takex ? 1 : 0;
                    yj += takex ? 0 : 1;
                }
            }
        }
        __syncthreads();
        // emission flags (see the header)
        uint32_t emit = 0;
        if (dt < m) {
#pragma unroll
            for (int q = 0; q < kSetItems; q++) {
                const int pos = dt + q;
                if (pos >= m)
                    break;
                const int e = msrc[pos];
                const bool ex = e < nX;
                bool f;
                if (S.op == 0) {                     // UNION
                    const bool hp = pos > 0 || nbr[0];
                    const int pr = pos > 0 ? msrc[pos - 1] : kSetT;
                    f = !(hp && scmp<NC>(s, pr, e) == 0);
                } else if (S.op == 1) {              // INTERSECT
                    const bool hp = pos > 0 || nbr[0];
                    const int pr = pos > 0 ? msrc[pos - 1] : kSetT;
                    const bool prx = pos > 0 ? (pr < nX) : (nbr[1] != 0);
                    f = !ex && hp && prx && scmp<NC>(s, pr, e) == 0;
                } else {                             // DIFFERENCE x - y
                    const bool hs = pos + 1 < m || nbr[2];
                    const int sc = pos + 1 < m ? msrc[pos + 1] : kSetT + 1;
                    f = ex && !(hs && scmp<NC>(s, sc, e) == 0);
                }
                emit |= (uint32_t)f << q;
            }
        }
        // block exclusive scan of the per-thread emission counts (thread order = merged order)
        const int cnt = __popc(emit);
        int inc = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += y;
        }
        if (lane == 31)
            wcnt[warp] = inc;
        __syncthreads();
        int base = 0, tot = 0;
        for (int w = 0; w < kThreads / 32; w++) {
            if (w < warp) base += wcnt[w];
            tot += wcnt[w];
        }
        base += inc - cnt;
        if (!WRITE) {
            if (tid == 0)
                S.pcount[p] = (uint64_t)tot;
            continue;
        }
        int64_t o;
        if (S.status) {
            // single pass: decoupled look-back over the partitions (claimed in order)
            if (warp == 0) {
                const uint64_t excl = lookback_warp(S.status, p, (uint64_t)tot, S.epoch);
                if (lane == 0) {
                    pbase = (int64_t)excl;
                    if (p == S.nparts - 1)
                        *S.total = (int64_t)excl + tot;
                }
            }
            __syncthreads();
            o = pbase + base;
        } else {
            o = (int64_t)S.pcount[p] + base;
        }
        for (uint32_t em = emit; em; em &= em - 1) {
            const int q = __ffs(em) - 1;
            const int e = msrc[dt + q];
            if (o < S.cap) {
                if (PACKED)
                    store_packed(S, o, s[e]);
                else
                    for (int c = 0; c < nc; c++)
                        store_okey(S.out[c], S.types[c], o, s[c * kSetS + e]);
            }
            o++;
        }
    }
    if (claim)
        cta_exit_reset(S.ctrs);
}

// exclusive scan of the per-partition counts (one CTA) and the total
__global__ void __launch_bounds__(1024) k_set_scan(const __grid_constant__ SetLaunch S)
{
    __shared__ uint64_t ws[32];
    __shared__ uint64_t carry;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0)
        carry = 0;
    __syncthreads();
    for (int64_t b0 = 0; b0 < S.nparts; b0 += 1024) {
        const int64_t p = b0 + tid;
        const uint64_t v = p < S.nparts ? S.pcount[p] : 0;
        uint64_t x = v;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint64_t y = __shfl_up_sync(0xffffffffu, x, d);
            if (lane >= d) x += y;
        }
        if (lane == 31)
            ws[warp] = x;
        __syncthreads();
        if (warp == 0) {
            uint64_t w = ws[lane];
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint64_t y = __shfl_up_sync(0xffffffffu, w, d);
                if (lane >= d) w += y;
            }
            ws[lane] = w;
        }
        __syncthreads();
        if (p < S.nparts)
            S.pcount[p] = carry + (warp ? ws[warp - 1] : 0) + x - v;
        __syncthreads();
        if (tid == 0)
            carry += ws[31];
        __syncthreads();
    }
    if (tid == 0)
        *S.total = (int64_t)carry;
}

size_t set_op_smem(int ncols) { return (size_t)ncols * kSetS * 8 + (size_t)kSetT * 4; }
int set_partition_rows() { return kSetT; }

template <int NC, bool PACKED>
static void set_passes(const SetLaunch &S, int sms, cudaStream_t st)
{
    const size_t smem = set_op_smem(NC);
    cudaFuncSetAttribute(k_set_op<NC, false, PACKED>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_set_op<NC, true, PACKED>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_set_op<NC, true, PACKED>, kThreads, smem);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(S.nparts, (int64_t)sms * std::max(occ, 1)));
    if (S.status) {                       // single pass with decoupled look-back
        if (S.nparts > 0)
            k_set_op<NC, true, PACKED><<<grid, kThreads, smem, st>>>(S);
        else
            cudaMemsetAsync(S.total, 0, sizeof(int64_t), st);
        return;
    }
    if (S.nparts > 0)
        k_set_op<NC, false, PACKED><<<grid, kThreads, smem, st>>>(S);
    k_set_scan<<<1, 1024, 0, st>>>(S);
    if (S.nparts > 0)
        k_set_op<NC, true, PACKED><<<grid, kThreads, smem, st>>>(S);
}

cudaError_t set_op_launch(const SetLaunch &S, int sms, cudaStream_t st)
{
    k_set_splits<<<(unsigned)((S.nparts + 1 + 255) / 256), 256, 0, st>>>(S);
    int bytes = 0;
    for (int c = 0; c < S.ncols; c++)
        bytes += type_width(S.types[c]);
    if (bytes <= 8) {
        set_passes<1, true>(S, sms, st);      // one packed u64 per tuple
        return cudaGetLastError();
    }
    switch (S.ncols) {
    case 2: set_passes<2, false>(S, sms, st); break;
    case 3: set_passes<3, false>(S, sms, st); break;
    default: set_passes<4, false>(S, sms, st); break;
    }
    return cudaGetLastError();
}

}  // namespace rw
