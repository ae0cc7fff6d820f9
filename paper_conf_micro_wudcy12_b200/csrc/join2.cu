// join2.cu — the sorted-key JOIN hot path (§4.3.2,
// Fig. 13; Fig. 14(b)), rebuilt as three kernels with no host synchronisation:
//
//   k_jsplit<K>      merge-path split of every partition boundary of A ∪ B (keys in
//                    order-preserving unsigned images, A first on ties);
//   k_jmatch<K>      ONE pass over the keys: per partition, the merged walk finds the
//                    head of every key segment [A rows][B rows]; a key with rows on both
//                    sides is a matched run (first rows, lengths, candidate count
//                    weight(a) * lenB); two decoupled look-backs (runs, candidates) give
//                    every run its record index and its output offset.  Chained for a
//                    3-input JOIN -> JOIN (Fig. 14(b)): the A side is then the list of
//                    first-level runs (unique keys, weight lenA * lenB) and the records
//                    written are the composed (a, b, c) runs;
//   k_jtiles         first run of every expansion tile (tile_run[t]), sized from the
//                    device-resident candidate total;
//   k_join_emit      output-balanced expansion: tile t holds candidates [t*T, t*T+T)
//                    of the join in (key, a, b, c) order; each candidate is mapped to its
//                    run and (i, j, k) in mixed radix (lenB, lenC), the live columns are
//                    gathered into the tile, and the fused downstream SELECT / PROJECT
//                    program, compaction, look-back and store run as in scan_emit.cu.
//                    The producer warp stages each tile's run records with TMA bulk copies.
#include "chain4.cuh"
#include "kernels.h"

namespace rw {

// ---------------------------------------------------------------------------
// keys: order-preserving unsigned image of the leading nkey columns (A6: sorted in
// each column's declared signedness, lexicographically)
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t col_img(const void *c, int type, int64_t i)
{
    switch (type) {
    case T_I32: return (uint32_t)((const int32_t *)c)[i] ^ 0x80000000u;
    case T_U32: return ((const uint32_t *)c)[i];
    case T_I64: return (uint64_t)((const int64_t *)c)[i] ^ 0x8000000000000000ull;
    case T_U64: return ((const uint64_t *)c)[i];
    default: return ((const uint8_t *)c)[i];
    }
}

template <typename K>
__device__ __forceinline__ K key_img(const KeySrc &S, int64_t i)
{
    if (S.img)
        return ((const K *)S.img)[i];
    uint64_t v = col_img(S.col[0], S.type[0], i);
    if (S.ncol == 2)
        v = (v << 32) | col_img(S.col[1], S.type[1], i);
    return (K)v;
}

// first index in [lo, n) whose key is > k (keys[lo - 1] <= k), galloping then bisection
template <typename K>
__device__ int64_t gallop_gt(const KeySrc &S, int64_t lo, int64_t n, K k)
{
    int64_t hi = n, step = 1;
    while (true) {
        const int64_t probe = lo + step - 1;
        if (probe >= n) { hi = n; break; }
        if (key_img<K>(S, probe) > k) { hi = probe; break; }
        lo = probe + 1;
        step <<= 1;
    }
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (key_img<K>(S, mid) <= k) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

constexpr int kMatchThreads = 256;
constexpr int kMatchItems = 16;
constexpr int kMatchT = kMatchThreads * kMatchItems;     // merged keys per partition

int match_partition() { return kMatchT; }

// A's row count is on the device for a chained match (the first-level run count)
__device__ __forceinline__ int64_t match_na(const MatchLaunch &M) { return M.nA_dev ? *M.nA_dev : M.nA; }

template <typename K>
__global__ void k_jsplit(const __grid_constant__ MatchLaunch M)
{
    const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nA = match_na(M);
    const int64_t nparts = (nA + M.nB + kMatchT - 1) / kMatchT;
    if (p > nparts)
        return;
    const int64_t d = min(p * kMatchT, nA + M.nB);
    int64_t lo = d > M.nB ? d - M.nB : 0, hi = d < nA ? d : nA;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (key_img<K>(M.A, mid) <= key_img<K>(M.B, d - mid - 1)) lo = mid + 1;
        else hi = mid;
    }
    M.split[p] = lo;
}

template <typename K>
__device__ __forceinline__ bool key_pass(const MatchLaunch &M, K k)
{
    bool ok = true;
    for (int i = 0; i < M.nkpred; i++) {
        const K c = (K)M.kpk[i];
        switch (M.kop[i]) {
        case C_LT: ok = ok && k < c; break;
        case C_LE: ok = ok && k <= c; break;
        case C_GT: ok = ok && k > c; break;
        case C_GE: ok = ok && k >= c; break;
        case C_EQ: ok = ok && k == c; break;
        default: ok = ok && k != c; break;
        }
    }
    return ok;
}

// One CTA per partition (claimed in order, so the look-backs always progress).
// RAW: the key is one 4- or 8-byte column; its slice is loaded with 16-byte vectors
// (the sign bit flipped for signed types); else the images are built element-wise.
template <typename K>
__host__ __device__ constexpr size_t match_smem() { return 2 * (size_t)(kMatchT + 8) * sizeof(K) + 2 * (size_t)kMatchT * 2 + 64; }

template <typename K, bool RAW>
__device__ __forceinline__ K *stage_keys(const KeySrc &S, int64_t i0, int64_t n_here, int64_t ntotal, K *raw)
{
    const int tid = threadIdx.x;
    const int64_t n_load = min(n_here + 1, ntotal - i0);        // + the first key past the partition
    if constexpr (RAW) {
        // 16-byte vectors of the aligned span: a vector never crosses a 16-byte boundary,
        // so the (unused) bytes read past the column's end stay inside its allocation
        constexpr int V = 16 / sizeof(K);
        const int64_t i0a = i0 & ~(int64_t)(V - 1);
        const int nvec = (int)((i0 + n_load - i0a + V - 1) / V);
        const K flip = S.type[0] == T_I32 || S.type[0] == T_I64 ? (K)((K)1 << (8 * sizeof(K) - 1)) : (K)0;
        const uint4 *src = (const uint4 *)((const K *)S.col[0] + i0a);
        for (int v = tid; v < nvec; v += kMatchThreads) {
            uint4 x = src[v];
            K *e = (K *)&x;
#pragma unroll
            for (int q = 0; q < V; q++)
                e[q] ^= flip;
            ((uint4 *)raw)[v] = x;
        }
        return raw + (i0 - i0a);
    } else {
        if (S.img && ((uintptr_t)S.img & 15) == 0) {
            // precomputed images (a chained match's first-level run keys): the same
            // 16-byte vector staging, no sign flip
            constexpr int V = 16 / sizeof(K);
            const int64_t i0a = i0 & ~(int64_t)(V - 1);
            const int nvec = (int)((i0 + n_load - i0a + V - 1) / V);
            const uint4 *src = (const uint4 *)((const K *)S.img + i0a);
            for (int v = tid; v < nvec; v += kMatchThreads)
                ((uint4 *)raw)[v] = src[v];
            return raw + (i0 - i0a);
        }
        if (!S.img && S.ncol == 1 && type_width(S.type[0]) == (int)sizeof(K) && ((uintptr_t)S.col[0] & 15) == 0) {
            // one raw key column of the image width (the other side of a chained match)
            constexpr int V = 16 / sizeof(K);
            const int64_t i0a = i0 & ~(int64_t)(V - 1);
            const int nvec = (int)((i0 + n_load - i0a + V - 1) / V);
            const K flip = S.type[0] == T_I32 || S.type[0] == T_I64 ? (K)((K)1 << (8 * sizeof(K) - 1)) : (K)0;
            const uint4 *src = (const uint4 *)((const K *)S.col[0] + i0a);
            for (int v = tid; v < nvec; v += kMatchThreads) {
                uint4 x = src[v];
                K *e = (K *)&x;
#pragma unroll
                for (int q = 0; q < V; q++)
                    e[q] ^= flip;
                ((uint4 *)raw)[v] = x;
            }
            return raw + (i0 - i0a);
        }
        // element-wise images, 4 loads in flight per thread
        int r = tid;
        for (; r + 3 * kMatchThreads < n_load; r += 4 * kMatchThreads) {
            K x[4];
#pragma unroll
            for (int u = 0; u < 4; u++)
                x[u] = key_img<K>(S, i0 + r + u * kMatchThreads);
#pragma unroll
            for (int u = 0; u < 4; u++)
                raw[r + u * kMatchThreads] = x[u];
        }
        for (; r < n_load; r += kMatchThreads)
            raw[r] = key_img<K>(S, i0 + r);
        return raw;
    }
}

template <typename K, bool RAW>
__global__ void __launch_bounds__(kMatchThreads, 4) k_jmatch(const __grid_constant__ MatchLaunch M)
{
    constexpr int NW = kMatchThreads / 32;
    constexpr K KMAX = (K)~(K)0;
    extern __shared__ __align__(16) unsigned char msm[];
    K *rawA = (K *)msm;
    K *rawB = rawA + (kMatchT + 8);
    uint16_t *hpos = (uint16_t *)(rawB + (kMatchT + 8));
    uint16_t *hia = hpos + kMatchT;
    __shared__ uint32_t wsum[NW];
    __shared__ uint32_t wrun[NW];
    __shared__ uint64_t wcand[NW];
    __shared__ int64_t sp, base_run;
    __shared__ uint64_t base_cand;
    __shared__ uint32_t last_la, last_lb;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0)
        sp = (int64_t)atomicAdd(&M.ctrs[0], 1u);
    __syncthreads();
    const int64_t p = sp;
    const int64_t NA = match_na(M);
    const int64_t nparts = (NA + M.nB + kMatchT - 1) / kMatchT;
    if (p >= nparts) {                          // chained match: fewer partitions than launched
        if (p == 0 && tid == 0) {
            M.totals[0] = 0;
            M.totals[1] = 0;
        }
        cta_exit_reset(M.ctrs);
        return;
    }
    const int64_t ntot = NA + M.nB;
    const int64_t d0 = p * kMatchT, d1 = min(d0 + kMatchT, ntot);
    const int64_t i0 = M.split[p], i1 = M.split[p + 1], j0 = d0 - i0, j1 = d1 - i1;
    const int nA = (int)(i1 - i0), nB = (int)(j1 - j0), m = (int)(d1 - d0);
    const K *sA = stage_keys<K, RAW>(M.A, i0, nA, NA, rawA);
    const K *sB = stage_keys<K, RAW>(M.B, j0, nB, M.nB, rawB);
    // merged predecessor of the partition (larger of the preceding A / B keys)
    bool p_has = false;
    K p_key = 0;
    if (i0 > 0) { p_key = key_img<K>(M.A, i0 - 1); p_has = true; }
    if (j0 > 0) { const K b = key_img<K>(M.B, j0 - 1); p_key = p_has && p_key > b ? p_key : b; p_has = true; }
    __syncthreads();

    // 1. merge walk over the thread's positions: segment heads, and which side each
    //    position comes from (A first on ties)
    uint32_t hbits = 0, abits = 0;
    int ia0 = 0;
    const int dt = tid * kMatchItems;
    if (dt < m) {
        int lo = dt > nB ? dt - nB : 0, hi = dt < nA ? dt : nA;
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (sA[mid] <= sB[dt - mid - 1]) lo = mid + 1;
            else hi = mid;
        }
        ia0 = lo;
        int ia = lo, jb = dt - lo;
        bool has_prev = dt > 0 || p_has;
        K prev = p_key;
        if (dt > 0) {
            prev = ia > 0 ? sA[ia - 1] : (K)0;
            if (jb > 0) { const K b = sB[jb - 1]; prev = ia > 0 && prev > b ? prev : b; }
        }
        K ca = ia < nA ? sA[ia] : KMAX, cb = jb < nB ? sB[jb] : KMAX;
        // branch-free steps (no divergence between lanes taking A and B): positions past
        // the partition's end (last partition only) are cleared from the masks after
        const uint32_t live = dt + kMatchItems <= m ? 0xffffffffu : ((1u << (m - dt)) - 1u);
        if (!has_prev)
            prev = ca < cb || (ca == cb && ia < nA) ? ca + 1 : cb + 1;   // any value != the first key
#pragma unroll
        for (int q = 0; q < kMatchItems; q++) {
            const bool takeA = ca < cb || (ca == cb && ia < nA);
            const K key = takeA ? ca : cb;
            hbits |= (uint32_t)(key != prev) << q;
            abits |= (uint32_t)takeA << q;
            prev = key;
            const int nx = takeA ? ia + 1 : jb + 1;
            const K v = takeA ? (nx < nA ? sA[nx] : KMAX) : (nx < nB ? sB[nx] : KMAX);
            ia += takeA ? 1 : 0;
            jb += takeA ? 0 : 1;
            ca = takeA ? v : ca;
            cb = takeA ? cb : v;
        }
        hbits &= live;
        abits &= live;
    }
    // 2. heads, in merged order, into smem (position and A index)
    const int nh = __popc(hbits);
    int hinc = nh;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, hinc, o);
        if (lane >= o) hinc += y;
    }
    if (lane == 31)
        wsum[warp] = (uint32_t)hinc;
    __syncthreads();
    int hb = 0, H = 0;
#pragma unroll
    for (int w = 0; w < NW; w++) {
        hb += w < warp ? (int)wsum[w] : 0;
        H += (int)wsum[w];
    }
    hb += hinc - nh;
    for (uint32_t hm = hbits; hm; hm &= hm - 1) {
        const int q = __ffs(hm) - 1;
        hpos[hb] = (uint16_t)(dt + q);
        hia[hb] = (uint16_t)(ia0 + __popc(abits & ((1u << q) - 1u)));
        hb++;
    }
    __syncthreads();
    // 3. runs of the thread's heads (blocked, balanced): lengths from the next head; the
    //    last head's segment may continue past the partition (galloped once, kept)
    const int per = (H + kMatchThreads - 1) / kMatchThreads;
    const int k0 = min(H, tid * per), k1 = min(H, k0 + per);
    if (k1 == H && k0 < k1) {
        const int k = H - 1, ia = hia[k], jb = hpos[k] - ia;
        const K key = ia < nA ? sA[ia] : sB[jb];
        int64_t ea = nA, eb = nB;
        if (i1 < NA && sA[nA] == key)
            ea = gallop_gt<K>(M.A, i1 + 1, NA, key) - i0;
        if (j1 < M.nB && sB[nB] == key)
            eb = gallop_gt<K>(M.B, j1 + 1, M.nB, key) - j0;
        last_la = (uint32_t)(ea - ia);
        last_lb = (uint32_t)(eb - jb);
    }
    __syncthreads();
    auto lens = [&](int k, uint32_t &la, uint32_t &lb) {
        const int ia = hia[k], jb = hpos[k] - ia;
        if (k + 1 < H) {
            la = (uint32_t)(hia[k + 1] - ia);
            lb = (uint32_t)(hpos[k + 1] - hia[k + 1] - jb);
        } else {
            la = last_la;
            lb = last_lb;
        }
    };
    // heads in batches of 4: a chained match's weight loads (global) are all in flight
    // before any is used
    constexpr int HB = 4;
    uint32_t nrun = 0;
    uint64_t ncand = 0;
    for (int kb = k0; kb < k1; kb += HB) {
        uint32_t lb[HB];
        uint64_t w[HB];
        bool ok[HB];
#pragma unroll
        for (int u = 0; u < HB; u++) {
            const int k = kb + u;
            uint32_t la = 0;
            lb[u] = 0;
            ok[u] = false;
            w[u] = 0;
            if (k < k1) {
                lens(k, la, lb[u]);
                const int ia = hia[k];
                ok[u] = la > 0 && lb[u] > 0 && key_pass<K>(M, sA[ia]);
                w[u] = M.wA ? (ok[u] ? __ldg(M.wA + i0 + ia) : 0ull) : (uint64_t)la;
            }
        }
#pragma unroll
        for (int u = 0; u < HB; u++)
            if (ok[u]) {
                nrun++;
                ncand += w[u] * lb[u];
            }
    }
    // 4. block exclusive scan of (runs, candidates) in head order
    uint32_t ir = nrun;
    uint64_t ic = ncand;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t yr = __shfl_up_sync(0xffffffffu, ir, o);
        const uint64_t yc = __shfl_up_sync(0xffffffffu, ic, o);
        if (lane >= o) {
            ir += yr;
            ic += yc;
        }
    }
    if (lane == 31) {
        wrun[warp] = ir;
        wcand[warp] = ic;
    }
    __syncthreads();
    uint32_t br = 0, tr = 0;
    uint64_t bc = 0, tc = 0;
#pragma unroll
    for (int w = 0; w < NW; w++) {
        if (w < warp) {
            br += wrun[w];
            bc += wcand[w];
        }
        tr += wrun[w];
        tc += wcand[w];
    }
    br += ir - nrun;
    bc += ic - ncand;
    // 5. decoupled look-backs (runs: warp 0, candidates: warp 1) over the partitions
    if (warp == 0) {
        const uint64_t e = lookback_warp(M.st_runs, p, tr, M.ep_runs);
        if (lane == 0) {
            base_run = (int64_t)e;
            if (p == nparts - 1)
                M.totals[0] = (int64_t)(e + tr);
        }
    } else if (warp == 1) {
        const uint64_t e = lookback_warp(M.st_cands, p, tc, M.ep_cands);
        if (lane == 0) {
            base_cand = e;
            if (p == nparts - 1)
                M.totals[1] = (int64_t)(e + tc);
        }
    }
    __syncthreads();
    // 6. records of the matched runs, in key order (heads in batches of 4: every global
    //    load of a batch is issued before its records are stored)
    int64_t r = base_run + br;
    uint64_t off = base_cand + bc;
    for (int kb = k0; kb < k1; kb += HB) {
        uint32_t la[HB], lb[HB], x0[HB], x1[HB], x2[HB];
        uint64_t w[HB];
        int ia[HB], jb[HB];
        bool ok[HB];
#pragma unroll
        for (int u = 0; u < HB; u++) {
            const int k = kb + u;
            ok[u] = false;
            la[u] = lb[u] = x0[u] = x1[u] = x2[u] = 0;
            w[u] = 0;
            ia[u] = jb[u] = 0;
            if (k < k1) {
                lens(k, la[u], lb[u]);
                ia[u] = hia[k];
                jb[u] = hpos[k] - ia[u];
                ok[u] = la[u] > 0 && lb[u] > 0 && key_pass<K>(M, sA[ia[u]]);
                if (ok[u]) {
                    const int64_t ga = i0 + ia[u];
                    w[u] = M.wA ? __ldg(M.wA + ga) : (uint64_t)la[u];
                    if (M.chain1) {
                        // 3-input composition: A element ga = first-level run
                        x0[u] = __ldg(M.c_s0 + ga);
                        x1[u] = __ldg(M.c_s1 + ga);
                        x2[u] = __ldg(M.c_len1 + ga);
                    }
                }
            }
        }
#pragma unroll
        for (int u = 0; u < HB; u++) {
            if (!ok[u])
                continue;
            const int64_t ga = i0 + ia[u], gb = j0 + jb[u];
            if (r < M.cap_runs) {
                if (M.chain1) {
                    M.s0[r] = x0[u];
                    M.s1[r] = x1[u];
                    M.len1[r] = x2[u];
                    M.s2[r] = (uint32_t)gb;
                    M.len2[r] = lb[u];
                } else {
                    M.s0[r] = (uint32_t)ga;
                    M.s1[r] = (uint32_t)gb;
                    M.len1[r] = lb[u];
                    if (M.len0) M.len0[r] = la[u];
                    if (M.key_out) ((K *)M.key_out)[r] = sA[ia[u]];
                    if (M.w_out) M.w_out[r] = (uint64_t)la[u] * lb[u];
                }
                M.off[r] = off;
            }
            r++;
            off += w[u] * lb[u];
        }
    }
    cta_exit_reset(M.ctrs);
}

// first run of every expansion tile: tile_run[t] = (last run with off <= t*T),
// t = 0 .. ntiles (entry ntiles = nruns - 1); ntiles from the device-resident total
__global__ void k_jtiles(const uint64_t *off, const int64_t *totals, int64_t T, int64_t cap_tiles, int64_t *tile_run,
                         int32_t *overflow)
{
    const int64_t nruns = totals[0], total = totals[1];
    const int64_t ntiles = (total + T - 1) / T;
    if (ntiles + 1 > cap_tiles) {
        if (blockIdx.x == 0 && threadIdx.x == 0)
            *overflow = 1;
        return;
    }
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t <= ntiles; t += (int64_t)gridDim.x * blockDim.x) {
        if (t == ntiles) {
            tile_run[t] = nruns - 1;
            continue;
        }
        const uint64_t o = (uint64_t)(t * T);
        int64_t lo = 0, hi = nruns;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (off[mid] <= o) lo = mid + 1;
            else hi = mid;
        }
        tile_run[t] = lo - 1;
    }
}

// ===========================================================================
// Expansion fused with the downstream chain
// ===========================================================================
constexpr int kJMaxStages = 4;
constexpr uint32_t kJBar = 1;             // named barrier of the compute warps
constexpr int kJWriters = 4;
constexpr int kJAux = 32 * (1 + kJWriters);
constexpr int kJSlots = 16;
constexpr int kEmitCnt = 32;
constexpr int kJRegCols = 4;              // register gather path: <= 4 live columns of 1 or 4 bytes

struct JBlk {
    uint64_t aggr, oempty;
    int64_t tile;
    uint32_t total, roff, used, br;
};

struct JCtl {
    uint64_t full[kJMaxStages], empty[kJMaxStages];
    int64_t tile[kJMaxStages];
    int64_t r0[kJMaxStages];              // first run of the tile
    int32_t rsh[kJMaxStages];             // r0 - (staged base run)
    int32_t nrec[kJMaxStages];            // runs overlapping the tile
    JBlk blk[kJSlots];
    uint32_t cnt[2][kEmitCnt];
    uint32_t wmax[32];
    volatile uint32_t tail;
};

static __host__ __device__ inline size_t al128j(size_t x) { return (x + 127) / 128 * 128; }
__device__ __forceinline__ uint32_t al16j(uint32_t x) { return (x + 15u) & ~15u; }

size_t join_emit_ctl_bytes() { return al128j(sizeof(JCtl)); }

// a tile of T candidates overlaps at most T runs; staged from a 4-aligned base run,
// rounded up to 4: <= T + 6 entries per record array
uint32_t join_rec_cap4(int T) { return (uint32_t)((T + 8 + 3) & ~3); }
size_t join_rec_stage_bytes(int ways, int T)
{
    const size_t n = join_rec_cap4(T);
    return al128j(n * 8) + (ways == 3 ? 5 : 3) * al128j(n * 4);
}

template <typename T>
__device__ __forceinline__ void emit_copy_j(T *dst, const T *src, int64_t base, uint32_t total, int64_t cap, int lane)
{
    const int64_t lim = cap - base;
    const uint32_t m = (int64_t)total < lim ? total : (lim > 0 ? (uint32_t)lim : 0u);
    T *d = dst + base;
    uint32_t j0 = 0;
    if (sizeof(T) >= 4) {
        constexpr int V = 16 / sizeof(T);
        const uint4 *s4 = (const uint4 *)src;
        const uint32_t nv = m / V;
        for (uint32_t j = lane; j < nv; j += 32) {
            const uint4 v = s4[j];
            const T *e = (const T *)&v;
#pragma unroll
            for (int x = 0; x < V; x++)
                d[(size_t)j * V + x] = e[x];
        }
        j0 = nv * V;
    }
    for (uint32_t j = j0 + lane; j < m; j += 32)
        d[j] = src[j];
}

__device__ __forceinline__ uint64_t gather_u(const void *col, int w, uint64_t row)
{
    if (w == 4) return __ldg((const uint32_t *)col + row);
    if (w == 8) return __ldg((const unsigned long long *)col + row);
    return __ldg((const uint8_t *)col + row);
}

// Unsigned 32-bit division by a run length via a multiply-high magic number (round-up
// method, exact for every 32-bit dividend): (m, s-1) with s = ceil(log2 l); l = 1 -> s = 0.
__device__ __forceinline__ uint2 fastdiv_magic(uint32_t l)
{
    if (l <= 1)
        return make_uint2(0u, 0xffffffffu);
    const uint32_t sft = 32 - __clz(l - 1);
    const uint64_t m = ((((uint64_t)1 << sft) - l) << 32) / l + 1;
    return make_uint2((uint32_t)m, sft - 1);
}
__device__ __forceinline__ uint32_t fastdiv(uint32_t d, uint2 mg)
{
    if (mg.y == 0xffffffffu)
        return d;
    const uint32_t hi = __umulhi(d, mg.x);
    return (hi + ((d - hi) >> 1)) >> mg.y;
}

template <int NT, int ITEMS, int WAYS, bool AGG = false>
__global__ void __launch_bounds__(NT + kJAux, 1) k_join_emit(const __grid_constant__ ChainProg P,
                                                           const __grid_constant__ TileLaunch L,
                                                           const __grid_constant__ JoinEmit X)
{
    constexpr int G = ITEMS / 4;
    constexpr int T = NT * ITEMS;
    constexpr int NW = NT / 32;
    static_assert(ITEMS % 4 == 0 && G <= 4 && G * NW <= kEmitCnt, "join tile geometry");
    extern __shared__ __align__(128) unsigned char smem_raw[];
    JCtl *ctl = (JCtl *)smem_raw;
    const int S = L.stages;
    const uint32_t RSB = X.rec_stage_bytes;
    char *rstage = (char *)smem_raw + al128j(sizeof(JCtl));
    char *tbuf = rstage + (size_t)S * RSB;                       // 2 gathered tiles (parity)
    uint32_t *rowbuf = (uint32_t *)(tbuf + 2 * (size_t)P.stage_bytes);   // candidate rows per side
    uint16_t *runidx = (uint16_t *)(rowbuf + (size_t)(WAYS == 3 ? 3 : 2) * T);   // candidate -> run
    char *scratch = (char *)(runidx + T);
    // aggregate terminal (JOIN -> chain -> AGG): the CTA's 128-bit accumulators instead of a ring
    unsigned long long *cta_acc = (unsigned long long *)(scratch + P.scratch_bytes);
    char *ring = scratch + P.scratch_bytes;
    const uint32_t R = L.out_bytes;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t total = *L.n_ptr;                              // join candidates (device)
    const int64_t ntiles = (total + T - 1) / T;
    // staged record arrays of stage s: off (u64), s0, s1, len1 [, s2, len2] (u32)
    const uint32_t cap4 = X.rec_cap4;                            // entries per staged array
    auto rec_off = [&](int s) { return (const uint64_t *)(rstage + (size_t)s * RSB); };
    auto rec_u32 = [&](int s, int a) {
        return (const uint32_t *)(rstage + (size_t)s * RSB + al128j((size_t)cap4 * 8) + (size_t)a * al128j((size_t)cap4 * 4));
    };

    if (tid == 0) {
        for (int s = 0; s < S; s++) {
            mbar_init(&ctl->full[s], 1);
            mbar_init(&ctl->empty[s], NW);
        }
        for (int j = 0; j < kJSlots; j++) {
            mbar_init(&ctl->blk[j].aggr, NW);
            mbar_init(&ctl->blk[j].oempty, 1);
        }
        ctl->tail = 0;
        fence_mbar_init();
    }
    if (AGG && P.agg_mode == 2)          // (global-atomic terminal: no CTA accumulators)
        for (int q = tid; q < P.D * (P.nagg + 1) * 2; q += blockDim.x)
            cta_acc[q] = 0;
    __syncthreads();

    if (warp == NW) {
        // ---------------- producer: claim tiles, stage their run records ----------------
        if (lane == 0) {
            int64_t tn = (int64_t)atomicAdd(&L.ctrs[0], 1u);
            int s = 0;
            uint32_t eph = 1;
            for (uint32_t i = 0;; ++i) {
                const int64_t t = tn;
                if (t < ntiles)
                    tn = (int64_t)atomicAdd(&L.ctrs[0], 1u);
                if (i >= (uint32_t)S)
                    mbar_wait(&ctl->empty[s], eph);
                ctl->tile[s] = t;
                if (t < ntiles) {
                    const int64_t r0 = X.tile_run[t], r1 = X.tile_run[t + 1];
                    const int64_t rb = r0 & ~(int64_t)3;
                    const uint32_t n4 = (uint32_t)(((r1 + 1 - rb) + 3) & ~(int64_t)3);
                    ctl->r0[s] = r0;
                    ctl->rsh[s] = (int32_t)(r0 - rb);
                    ctl->nrec[s] = (int32_t)(r1 - r0 + 1);
                    char *st = rstage + (size_t)s * RSB;
                    const int na = WAYS == 3 ? 5 : 3;
                    fence_proxy_async_smem();
                    mbar_arrive_expect_tx(&ctl->full[s], n4 * 8 + na * n4 * 4);
                    bulk_g2s_plain(st, X.off + rb, n4 * 8, &ctl->full[s]);
                    const uint32_t *src[5] = {X.s0, X.s1, X.len1, X.s2, X.len2};
                    for (int a = 0; a < na; a++)
                        bulk_g2s_plain(st + al128j((size_t)cap4 * 8) + (size_t)a * al128j((size_t)cap4 * 4), src[a] + rb,
                                       n4 * 4, &ctl->full[s]);
                } else {
                    mbar_arrive(&ctl->full[s]);
                    break;
                }
                if (++s == S) {
                    s = 0;
                    eph ^= 1u;
                }
            }
        }
    } else if (warp > NW) {
        // ---------------- writers: look-back + copy-out ----------------
        const int wi = warp - NW - 1;
        for (uint32_t i = wi;; i += kJWriters) {
            const int j = (int)(i % kJSlots);
            mbar_wait(&ctl->blk[j].aggr, (i / kJSlots) & 1u);
            const int64_t t = ctl->blk[j].tile;
            if (t >= ntiles)
                break;
            const uint32_t tot = ctl->blk[j].total;
            const int64_t excl = (int64_t)lookback_warp(L.status, t, tot, L.epoch, /*aggregate_published=*/true);
            if (lane == 0 && t == ntiles - 1)
                *L.n_dev = excl + (int64_t)tot;
            const uint32_t roff = ctl->blk[j].roff;
            uint32_t coff = 0;
            for (int c = 0; c < P.nout; c++) {
                const int w = P.out_w[c];
                // the ring is circular: a column's segment may wrap at R (16-byte aligned,
                // so no vector straddles the end) -> copied in two pieces
                const uint32_t so = roff + coff >= R ? roff + coff - R : roff + coff;   // roff, coff < R
                coff += al16j(tot * w);
                const uint32_t n1 = min(tot, (R - so) / (uint32_t)w);
                for (int piece = 0; piece < 2; piece++) {
                    const char *src = piece ? ring : ring + so;
                    const int64_t at = piece ? excl + n1 : excl;
                    const uint32_t cnt = piece ? tot - n1 : n1;
                    if (cnt == 0) continue;
                    if (w == 4) emit_copy_j<uint32_t>((uint32_t *)P.out_ptr[c], (const uint32_t *)src, at, cnt, P.out_capacity, lane);
                    else if (w == 8) emit_copy_j<uint64_t>((uint64_t *)P.out_ptr[c], (const uint64_t *)src, at, cnt, P.out_capacity, lane);
                    else emit_copy_j<uint8_t>((uint8_t *)P.out_ptr[c], (const uint8_t *)src, at, cnt, P.out_capacity, lane);
                }
            }
            __syncwarp();
            if (lane == 0) {
                if (i > 0)
                    mbar_wait(&ctl->blk[(i - 1) % kJSlots].oempty, ((i - 1) / kJSlots) & 1u);
                __threadfence_block();
                ctl->tail = ctl->tail + ctl->blk[j].used;
                mbar_arrive(&ctl->blk[j].oempty);
            }
            __syncwarp();
        }
    } else {
        // ---------------- compute warps ----------------
        // Per tile: (A) its gathered columns land (cp.async group) and are evaluated:
        // survivor counts, the count barrier, the tile aggregate is published; (B) the
        // next tile is filled: candidate -> run map (run starts scattered, block max-scan),
        // a fast-division magic per run, and the lane-strided gathers are issued (they fly
        // while (C) this tile is compacted into the ring).  The aggregate of a tile never
        // waits on the next tile's records.
        uint32_t head = 0, hpos = 0, ublk = 0;
        int s = 0;
        uint32_t fph = 0;
        uint32_t gv[kJRegCols][ITEMS];                  // register-gathered values of the next tile
        RegAgg racc;                                    // aggregate terminal: register partials
        int64_t since_flush = 0;
        if (AGG)
            reg_agg_zero(racc);
        char *pend_st = tbuf;
        int pend_rows = 0;
        auto fill = [&](uint32_t idx, int64_t &t) -> bool {
            mbar_wait(&ctl->full[s], fph);
            t = ctl->tile[s];
            if (t >= ntiles)
                return false;                           // the producer's sentinel
            char *st = tbuf + (size_t)(idx & 1u) * P.stage_bytes;
            const uint64_t c0g = (uint64_t)t * T;
            const int rows = (int)min((int64_t)T, total - (int64_t)c0g);
            const uint64_t *roff = rec_off(s);
            const uint32_t *rs0 = rec_u32(s, 0), *rs1 = rec_u32(s, 1), *rl1 = rec_u32(s, 2);
            const uint32_t *rs2 = rec_u32(s, 3), *rl2 = rec_u32(s, 4);
            const int sh = ctl->rsh[s], nrec = ctl->nrec[s];
            // (1) candidate -> run.  Few runs in the tile (long runs, e.g. Zipf hot keys):
            //     each thread binary-searches its first candidate over the staged run
            //     offsets (strictly increasing: every recorded run has >= 1 candidate) and
            //     walks forward, no block-wide step.  Many runs (short runs): run starts
            //     scattered into a cleared array, then a block max-scan.  (nrec is
            //     CTA-uniform, so is the branch.)
            uint16_t v[ITEMS];
            if (nrec <= T / 16) {
                const uint64_t cf = c0g + (uint64_t)(tid * ITEMS);
                int lo = 0, hi = nrec;                  // roff[sh + 0] <= c0g <= cf
                while (hi - lo > 1) {
                    const int mid = (lo + hi) >> 1;
                    if (roff[sh + mid] <= cf) lo = mid;
                    else hi = mid;
                }
                int r = lo;
                uint64_t nxt = r + 1 < nrec ? roff[sh + r + 1] : ~0ull;
#pragma unroll
                for (int k = 0; k < ITEMS; k++) {
                    while (cf + k >= nxt) {
                        ++r;
                        nxt = r + 1 < nrec ? roff[sh + r + 1] : ~0ull;
                    }
                    v[k] = (uint16_t)r;
                }
            } else {
#pragma unroll
                for (int k = 0; k < ITEMS; k += 4)
                    *(uint2 *)&runidx[tid * ITEMS + k] = make_uint2(0u, 0u);
                bar_sync(kJBar, NT);
                for (int rr = 1 + tid; rr < nrec; rr += NT) {
                    const uint64_t o = roff[sh + rr] - c0g;
                    if (o < (uint64_t)rows) runidx[o] = (uint16_t)rr;
                }
                bar_sync(kJBar, NT);
#pragma unroll
                for (int k = 0; k < ITEMS; k += 4) {
                    const uint2 x = *(const uint2 *)&runidx[tid * ITEMS + k];
                    v[k] = (uint16_t)x.x;
                    v[k + 1] = (uint16_t)(x.x >> 16);
                    v[k + 2] = (uint16_t)x.y;
                    v[k + 3] = (uint16_t)(x.y >> 16);
                }
#pragma unroll
                for (int k = 1; k < ITEMS; k++) v[k] = max(v[k], v[k - 1]);
                uint32_t mx = v[ITEMS - 1];
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, mx, o);
                    if (lane >= o) mx = max(mx, y);
                }
                if (lane == 31)
                    ctl->wmax[warp] = mx;
                const uint32_t before = __shfl_up_sync(0xffffffffu, mx, 1);
                bar_sync(kJBar, NT);
                uint32_t carry = lane > 0 ? before : 0u;
                for (int w = 0; w < warp; w++) carry = max(carry, ctl->wmax[w]);
#pragma unroll
                for (int k = 0; k < ITEMS; k++) v[k] = (uint16_t)max((uint32_t)v[k], carry);
            }
            // (2) thread-contiguous walk over candidates [tid*ITEMS, tid*ITEMS + ITEMS): rows
            //     of every candidate (a run change lands on (0, 0, 0)), into the row buffer
            const int cfirst = tid * ITEMS;
            const int nvalid = min(ITEMS, rows - cfirst);
            if (nvalid > 0) {
                int r = v[0];
                uint32_t l1 = rl1[sh + r], l2 = WAYS == 3 ? rl2[sh + r] : 1u;
                uint32_t b0 = rs0[sh + r], b1 = rs1[sh + r], b2 = WAYS == 3 ? rs2[sh + r] : 0u;
                uint64_t d = c0g + (uint64_t)cfirst - roff[sh + r];
                uint32_t ii, jj, kk = 0;
                if (WAYS == 3) {
                    const uint64_t qq = d / l2;
                    kk = (uint32_t)(d - qq * l2);
                    d = qq;
                }
                if (d <= 0xffffffffull) {
                    ii = (uint32_t)d / l1;
                    jj = (uint32_t)d - ii * l1;
                } else {
                    ii = (uint32_t)(d / l1);
                    jj = (uint32_t)(d - (uint64_t)ii * l1);
                }
                uint32_t ra[ITEMS], rb_[ITEMS], rc[WAYS == 3 ? ITEMS : 1];
#pragma unroll
                for (int q = 0; q < ITEMS; q++) {
                    if (q > 0 && v[q] != r) {
                        r = v[q];
                        l1 = rl1[sh + r];
                        b0 = rs0[sh + r];
                        b1 = rs1[sh + r];
                        if (WAYS == 3) {
                            l2 = rl2[sh + r];
                            b2 = rs2[sh + r];
                        }
                        ii = jj = kk = 0;
                    }
                    ra[q] = b0 + ii;
                    rb_[q] = b1 + jj;
                    if (WAYS == 3) {
                        rc[WAYS == 3 ? q : 0] = b2 + kk;
                        if (++kk == l2) {
                            kk = 0;
                            if (++jj == l1) { jj = 0; ++ii; }
                        }
                    } else if (++jj == l1) {
                        jj = 0;
                        ++ii;
                    }
                }
                if (nvalid == ITEMS) {
#pragma unroll
                    for (int q = 0; q < ITEMS; q += 4) {
                        *(uint4 *)&rowbuf[cfirst + q] = make_uint4(ra[q], ra[q + 1], ra[q + 2], ra[q + 3]);
                        *(uint4 *)&rowbuf[T + cfirst + q] = make_uint4(rb_[q], rb_[q + 1], rb_[q + 2], rb_[q + 3]);
                        if (WAYS == 3)
                            *(uint4 *)&rowbuf[2 * T + cfirst + q] =
                                make_uint4(rc[WAYS == 3 ? q : 0], rc[WAYS == 3 ? q + 1 : 0], rc[WAYS == 3 ? q + 2 : 0],
                                           rc[WAYS == 3 ? q + 3 : 0]);
                    }
                } else {
#pragma unroll
                    for (int q = 0; q < ITEMS; q++) {
                        if (q < nvalid) {
                            rowbuf[cfirst + q] = ra[q];
                            rowbuf[T + cfirst + q] = rb_[q];
                            if (WAYS == 3) rowbuf[2 * T + cfirst + q] = rc[WAYS == 3 ? q : 0];
                        }
                    }
                }
            }
            __syncwarp();
            // (3) gathers, lane-contiguous over the warp's candidates: consecutive lanes read
            //     consecutive rows of a run (coalesced) straight into the tile (cp.async); the
            //     column metadata (warp-uniform) is read once per tile
            {
                const uint32_t st_s = smem_u32(st);
                const int wbase = warp * 32 * ITEMS;
                uint32_t rA[ITEMS], rB[ITEMS], rC[WAYS == 3 ? ITEMS : 1];
#pragma unroll
                for (int q = 0; q < ITEMS; q++) {
                    const int cand = wbase + q * 32 + lane;
                    rA[q] = cand < rows ? rowbuf[cand] : 0u;
                    rB[q] = cand < rows ? rowbuf[T + cand] : 0u;
                    if (WAYS == 3) rC[WAYS == 3 ? q : 0] = cand < rows ? rowbuf[2 * T + cand] : 0u;
                }
                const int ncols = X.ncols;
                if (X.regpath) {
                    // plain loads into registers (a run's repeated left row is one broadcast
                    // sector; cp.async would serialise identical addresses), stored into the
                    // tile at the top of the next iteration, so they fly during compaction
                    // 3-input groups: the column's side and width are warp-uniform, selected
                    // once per column, so the row loop is a plain gather (rows past the
                    // tile's end read row 0 of their side, which exists since the tile is
                    // not empty; measured C5 7.95 -> 7.69 ms).  2-input groups keep the
                    // per-element form, which measured faster there (C3 5.20 vs 5.37 ms).
#define RW_JGATHER(T_, ROWS_)                                                              \
    {                                                                                      \
        const T_ *sp_ = (const T_ *)src;                                                   \
        _Pragma("unroll") for (int q = 0; q < ITEMS; q++) gv[cc][q] = (uint32_t)__ldg(sp_ + ROWS_[q]); \
    }
#pragma unroll
                    for (int cc = 0; cc < kJRegCols; cc++) {
                        if (cc >= ncols) break;
                        const char *src = (const char *)X.src[cc];
                        const int w = X.w[cc], side = X.side[cc];
                        if constexpr (WAYS == 3) {
                            if (w == 4) {
                                if (side == 0) RW_JGATHER(uint32_t, rA)
                                else if (side == 1) RW_JGATHER(uint32_t, rB)
                                else RW_JGATHER(uint32_t, rC)
                            } else {
                                if (side == 0) RW_JGATHER(uint8_t, rA)
                                else if (side == 1) RW_JGATHER(uint8_t, rB)
                                else RW_JGATHER(uint8_t, rC)
                            }
                        } else {
#pragma unroll
                            for (int q = 0; q < ITEMS; q++) {
                                const int cand = wbase + q * 32 + lane;
                                const uint32_t row = side == 0 ? rA[q] : rB[q];
                                gv[cc][q] = cand < rows ? (w == 4 ? __ldg((const uint32_t *)src + row) : (uint32_t)__ldg((const uint8_t *)src + row)) : 0u;
                            }
                        }
                    }
#undef RW_JGATHER
                    pend_st = st;
                    pend_rows = rows;
                }
                for (int cc = 0; cc < ncols && !X.regpath; cc++) {
                    const char *src = (const char *)X.src[cc];
                    const uint32_t dst = st_s + P.slot[cc].off;
                    const int w = X.w[cc], side = X.side[cc];
                    if (w == 4 && side == 0) {
#pragma unroll
                        for (int q = 0; q < ITEMS; q++) {
                            const int cand = wbase + q * 32 + lane;
                            if (cand < rows) cp_async_s<4>(dst + (uint32_t)cand * 4, src + (size_t)rA[q] * 4);
                        }
                    } else if (w == 4 && side == 1) {
#pragma unroll
                        for (int q = 0; q < ITEMS; q++) {
                            const int cand = wbase + q * 32 + lane;
                            if (cand < rows) cp_async_s<4>(dst + (uint32_t)cand * 4, src + (size_t)rB[q] * 4);
                        }
                    } else {
                        char *dp = st + P.slot[cc].off;
#pragma unroll
                        for (int q = 0; q < ITEMS; q++) {
                            const int cand = wbase + q * 32 + lane;
                            if (cand < rows) {
                                const uint32_t row = side == 0 ? rA[q] : side == 1 ? rB[q] : rC[WAYS == 3 ? q : 0];
                                if (w == 4) cp_async_s<4>(dst + (uint32_t)cand * 4, src + (size_t)row * 4);
                                else if (w == 8) cp_async_s<8>(dst + (uint32_t)cand * 8, src + (size_t)row * 8);
                                else dp[cand] = src[row];
                            }
                        }
                    }
                }
            }
            cp_async_commit();
            __syncwarp();
            if (lane == 0)
                mbar_arrive(&ctl->empty[s]);
            if (++s == S) {
                s = 0;
                fph ^= 1u;
            }
            return true;
        };
        int64_t t;
        bool have = fill(0, t);
        for (uint32_t i = 0; have; ++i) {
            if (X.regpath) {
                // the register-gathered values of tile i into its tile buffer
                const int wbase = warp * 32 * ITEMS;
#pragma unroll
                for (int cc = 0; cc < kJRegCols; cc++) {
                    if (cc >= X.ncols) break;
                    char *dst = pend_st + P.slot[cc].off;
                    if (X.w[cc] == 4) {
#pragma unroll
                        for (int q = 0; q < ITEMS; q++)
                            if (wbase + q * 32 + lane < pend_rows) ((uint32_t *)dst)[wbase + q * 32 + lane] = gv[cc][q];
                    } else {
#pragma unroll
                        for (int q = 0; q < ITEMS; q++)
                            if (wbase + q * 32 + lane < pend_rows) ((uint8_t *)dst)[wbase + q * 32 + lane] = (uint8_t)gv[cc][q];
                    }
                }
            } else {
                cp_async_wait_group<0>();
            }
            bar_sync(kJBar, NT);                        // tile i's gathers visible to every thread
            const int par = (int)(i & 1u);
            char *st = tbuf + (size_t)(i & 1u) * P.stage_bytes;
            const uint64_t c0g = (uint64_t)t * T;
            const int rows = (int)min((int64_t)T, total - (int64_t)c0g);
            uint32_t mask0 = 0;
#pragma unroll
            for (int g = 0; g < G; g++)
#pragma unroll
                for (int q = 0; q < 4; q++)
                    if (row4<NT>(g) + q < rows)
                        mask0 |= 1u << (g * 4 + q);
            const uint32_t m = run_ops4<NT, G>(P, 0, P.nops, st, scratch, mask0);
            if constexpr (AGG) {
                // aggregate terminal: every surviving candidate adds into the partials
                if (P.agg_mode == 2)
                    agg_tile_reg<NT, ITEMS, true>(P, st, scratch, m, racc, cta_acc, since_flush, L.err);
                else
                    agg_tile_global<NT, ITEMS, true>(P, st, scratch, m, L.agg_acc, L.err);
                int64_t tn;
                const bool next = fill(i + 1, tn);
                t = tn;
                have = next;
                continue;
            }
            uint32_t pk = 0;
#pragma unroll
            for (int g = 0; g < G; g++)
                pk |= (uint32_t)__popc((m >> (4 * g)) & 15u) << (8 * g);
            uint32_t inc = pk;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o)
                    inc += y;
            }
            if (lane == 31)
#pragma unroll
                for (int g = 0; g < G; g++)
                    ctl->cnt[par][g * NW + warp] = (inc >> (8 * g)) & 255u;
            const uint32_t ex = inc - pk;
            bar_sync(kJBar, NT);
            const uint32_t v = lane < G * NW ? ctl->cnt[par][lane] : 0u;
            uint32_t bin = v;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, bin, o);
                if (lane >= o)
                    bin += y;
            }
            const uint32_t tot = __shfl_sync(0xffffffffu, bin, 31);
            uint32_t pre[G];
#pragma unroll
            for (int g = 0; g < G; g++)
                pre[g] = __shfl_sync(0xffffffffu, bin - v, g * NW + warp) + ((ex >> (8 * g)) & 255u);
            if (warp == 0 && lane == 0 && t > 0)
                st_relaxed_u64(&L.status[t], ((uint64_t)L.epoch << 48) | (1ull << 46) | tot);
            int64_t tn;
            const bool next = fill(i + 1, tn);
            const uint32_t need = P.br_nw[0][0] * al16j(tot) + P.br_nw[0][1] * al16j(tot * 4u) + P.br_nw[0][2] * al16j(tot * 8u);
            // circular ring: a block may wrap at R; wait until its bytes are free
            const uint32_t pos = hpos, used = need;
            const int j = (int)(ublk % kJSlots);
            if (ublk >= kJSlots)
                mbar_wait(&ctl->blk[j].oempty, ((ublk / kJSlots) - 1) & 1u);
            {
                uint32_t backoff = 64;
                while (head + used - ctl->tail > R) {
                    __nanosleep(backoff);
                    backoff = backoff < 1024 ? backoff * 2 : 1024;
                }
            }
            head += used;
            hpos = pos + need >= R ? pos + need - R : pos + need;
            uint32_t sp[G][4];
#pragma unroll
            for (int g = 0; g < G; g++) {
                uint32_t p = pre[g];
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    sp[g][q] = p;
                    p += (m >> (4 * g + q)) & 1u;
                }
            }
            uint32_t coff = 0;
            for (int c = 0; c < P.nout; c++) {
                const int w = P.out_w[c];
                const char *src = loc_ptr(P.out_loc[c], st, scratch);
                const uint32_t so = pos + coff >= R ? pos + coff - R : pos + coff;   // pos, coff < R
                coff += al16j(tot * w);
                if (so + tot * (uint32_t)w > R) {
                    // this column's segment wraps at the ring's end: positions mod R
                    wrap_scatter<NT, G>(ring, R, so, w, src, m, sp);
                    continue;
                }
                char *d = ring + so;
#pragma unroll
                for (int g = 0; g < G; g++) {
                    const uint32_t m4 = (m >> (4 * g)) & 15u;
                    if (!m4)
                        continue;
                    if (w == 4) {
                        const V4<uint32_t> x = ld4<uint32_t>(src, row4<NT>(g));
#pragma unroll
                        for (int q = 0; q < 4; q++)
                            if ((m4 >> q) & 1u) ((uint32_t *)d)[sp[g][q]] = x.v[q];
                    } else if (w == 8) {
                        const V4<uint64_t> x = ld4<uint64_t>(src, row4<NT>(g));
#pragma unroll
                        for (int q = 0; q < 4; q++)
                            if ((m4 >> q) & 1u) ((uint64_t *)d)[sp[g][q]] = x.v[q];
                    } else {
                        const V4<uint8_t> x = ld4<uint8_t>(src, row4<NT>(g));
#pragma unroll
                        for (int q = 0; q < 4; q++)
                            if ((m4 >> q) & 1u) ((uint8_t *)d)[sp[g][q]] = x.v[q];
                    }
                }
            }
            __syncwarp();
            if (lane == 0) {
                if (warp == 0) {
                    ctl->blk[j].tile = t;
                    ctl->blk[j].total = tot;
                    ctl->blk[j].roff = pos;
                    ctl->blk[j].used = used;
                    ctl->blk[j].br = 0;
                }
                mbar_arrive(&ctl->blk[j].aggr);
            }
            ++ublk;
            t = tn;
            have = next;
        }
        if (AGG && P.agg_mode == 2)
            reg_agg_reduce_warp(P, racc, cta_acc);   // warp-reduced, 128-bit exact
        if (tid == 0) {
            for (uint32_t u = ublk; u < ublk + kJWriters; ++u) {
                const int ju = (int)(u % kJSlots);
                if (u >= kJSlots)
                    mbar_wait(&ctl->blk[ju].oempty, ((u / kJSlots) - 1) & 1u);
                ctl->blk[ju].tile = ntiles;
                mbar_arrive_cnt(&ctl->blk[ju].aggr, NW);
            }
        }
    }
    __syncthreads();
    if (AGG) {
        if (P.agg_mode == 2)
            for (int q = tid; q < P.D * (P.nagg + 1); q += blockDim.x) {
                const unsigned long long lo = cta_acc[2 * q], hi = cta_acc[2 * q + 1];
                if (lo | hi)
                    atomic_add128(&L.agg_acc[2 * q], &L.agg_acc[2 * q + 1], lo, hi);
            }
    } else if (blockIdx.x == 0 && tid == 0 && ntiles == 0) {
        *L.n_dev = 0;
    }
    cta_exit_reset(L.ctrs);
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
template <typename K, bool RAW>
static cudaError_t match_go(const MatchLaunch &M, cudaStream_t st)
{
    k_jsplit<K><<<(unsigned)((M.nparts + 1 + 255) / 256), 256, 0, st>>>(M);
    if (M.nparts > 0) {
        cudaFuncSetAttribute(k_jmatch<K, RAW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)match_smem<K>());
        k_jmatch<K, RAW><<<(unsigned)M.nparts, kMatchThreads, match_smem<K>(), st>>>(M);
    }
    return cudaGetLastError();
}

cudaError_t match_launch(const MatchLaunch &M, bool wide, cudaStream_t st)
{
    // raw vector staging: both sides one 4- or 8-byte column (not precomputed images)
    const bool raw = !M.A.img && !M.B.img && M.A.ncol == 1 && M.B.ncol == 1 && M.A.type[0] != T_U8;
    if (wide)
        return raw ? match_go<uint64_t, true>(M, st) : match_go<uint64_t, false>(M, st);
    return raw ? match_go<uint32_t, true>(M, st) : match_go<uint32_t, false>(M, st);
}

cudaError_t jtiles_launch(const uint64_t *off, const int64_t *totals, int64_t T, int64_t cap_tiles, int64_t *tile_run,
                          int32_t *overflow, int sms, cudaStream_t st)
{
    k_jtiles<<<sms * 4, 256, 0, st>>>(off, totals, T, cap_tiles, tile_run, overflow);
    return cudaGetLastError();
}

template <int NT, int ITEMS, int WAYS, bool AGG = false>
static int jocc(size_t smem)
{
    auto f = k_join_emit<NT, ITEMS, WAYS, AGG>;
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, f, NT + kJAux, smem) != cudaSuccess)
        return 0;
    return n;
}

int join_emit_occupancy(int nt, int items, int ways, size_t smem, bool agg)
{
    if (agg)
        return ways == 3 ? jocc<256, 8, 3, true>(smem) : jocc<256, 8, 2, true>(smem);
    if (nt == 512)
        return ways == 3 ? jocc<512, 4, 3>(smem) : jocc<512, 4, 2>(smem);
    if (ways == 3)
        return items == 4 ? jocc<256, 4, 3>(smem) : jocc<256, 8, 3>(smem);
    return items == 4 ? jocc<256, 4, 2>(smem) : jocc<256, 8, 2>(smem);
}

template <int NT, int ITEMS, int WAYS, bool AGG = false>
static cudaError_t jgo(const ChainProg &P, const TileLaunch &L, const JoinEmit &X, size_t smem, int grid, cudaStream_t s)
{
    cudaFuncSetAttribute(k_join_emit<NT, ITEMS, WAYS, AGG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    k_join_emit<NT, ITEMS, WAYS, AGG><<<grid, NT + kJAux, smem, s>>>(P, L, X);
    return cudaGetLastError();
}

cudaError_t join_emit_launch(const ChainProg &P, const TileLaunch &L, const JoinEmit &X, int nt, int items, int ways,
                             size_t smem, int grid, cudaStream_t s)
{
    if (P.is_agg)
        return ways == 3 ? jgo<256, 8, 3, true>(P, L, X, smem, grid, s) : jgo<256, 8, 2, true>(P, L, X, smem, grid, s);
    if (nt == 512)
        return ways == 3 ? jgo<512, 4, 3>(P, L, X, smem, grid, s) : jgo<512, 4, 2>(P, L, X, smem, grid, s);
    if (ways == 3)
        return items == 4 ? jgo<256, 4, 3>(P, L, X, smem, grid, s) : jgo<256, 8, 3>(P, L, X, smem, grid, s);
    return items == 4 ? jgo<256, 4, 2>(P, L, X, smem, grid, s) : jgo<256, 8, 2>(P, L, X, smem, grid, s);
}

}  // namespace rw
