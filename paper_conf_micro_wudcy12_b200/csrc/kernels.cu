// kernels.cu — the sm_100a kernels of the fused relational-algebra hot path.
//
//   k_scan_chain<ITEMS, AGG>  fused SELECT / PROJECT / arithmetic chain over one
//                             input relation, terminal =
//                             compacted store or group-by aggregate (a9).
//   k_agg_finalize            128-bit accumulators -> output relation (groups with
//                             count > 0, ascending code).
//   k_join_runs<K>            merge-path partitioned sorted-key JOIN, phase 1:
//                             matched key runs + output offsets (a7).
//   k_tile_runs               first run of every expansion tile.
//   k_scan_chain<..., JOIN>   JOIN phase 2: output-balanced expansion (join_fill)
//                             fused with the downstream SELECT / PROJECT chain (a8),
//                             same warp-specialised pipeline as the scan chain.
//
// Every persistent kernel claims tiles with a global atomic counter (so the
// decoupled look-back always has forward progress) and the last CTA to leave
// resets the counter for the next launch.
#include <type_traits>
#include "chain.cuh"
#include "kernels.h"

namespace rw {

static __host__ __device__ inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// ===========================================================================
// Fused scan chain, warp-specialised (kThreads compute threads + 3 warps):
//   producer warp  : claims tiles in order (global atomic) and stages each live
//                    column of the tile into smem with one TMA bulk copy
//                    (cp.async.bulk -> full[s]), S input stages deep;
//   compute warps  : run the fused micro-op program on the tile, ballot-compact,
//                    block-scan, publish the tile aggregate for the look-back at
//                    once, then scatter the survivors (tile-local order) into a
//                    byte-granular smem ring and release the input stage;
//   4 writer warps : round-robin over compacted tiles: decoupled look-back for
//                    the tile's global offset, coalesced copy of its columns to
//                    HBM, release of its ring bytes (in tile order).
// Phase timing (scripts/phases.py) showed the offset of a tile resolves ~4 us
// after its aggregate (waiting for straggling predecessors); a compacted tile
// only holds its actual bytes (~6 KB at 25 % survival instead of a 24 KB
// worst-case slot) while it waits, so enough tiles stay in flight per SM.
// ===========================================================================
constexpr int kWriterWarps = 4;
constexpr int kAuxThreads = 32 * (kWriterWarps + 1);      // writer warps + producer warp
// aggregate kernels have no compacted output: no writer warps, only the producer
__host__ __device__ constexpr int aux_threads(bool agg) { return agg ? 32 : kAuxThreads; }
constexpr int kRingSlots = 16;          // compacted tiles awaiting their offset, per CTA
constexpr uint32_t kComputeBar = 1;     // named barrier of the compute warps

struct InCtl {
    uint64_t full, empty;
    int64_t tile;
};
struct BlkCtl {
    uint64_t aggr, oempty;
    int64_t tile;
    uint32_t total;
    uint32_t roff;                       // byte offset of the block in the ring
    uint32_t used;                       // ring bytes consumed (block + skipped tail)
    uint32_t br;                         // branch of the block (input-dependence fusion)
};
template <int NT, int ITEMS>
struct ScanCtl {
    InCtl in[kMaxStages];
    BlkCtl blk[kRingSlots];
    uint32_t cnt[2][ITEMS * NT / 32];    // double-buffered: a warp may run one tile ahead
    uint32_t total;
    uint32_t roff;
    volatile uint32_t tail;              // ring bytes released by the writers (monotone, wraps)
    uint32_t head;                       // ring bytes reserved by the compute warps (monotone, wraps)
    uint32_t hpos;                       // next write position in [0, R)
};

__device__ __forceinline__ uint32_t al16(uint32_t x) { return (x + 15u) & ~15u; }

template <typename T>
__device__ __forceinline__ T ld_ring(const T *p, bool gring)
{
    return gring ? __ldcg(p) : *p;     // global ring: read through L2 (written by other warps)
}

template <typename T>
__device__ __forceinline__ void group_copy_out(T *dst, const T *src, int64_t base, uint32_t total, int64_t cap,
                                               int q, int nq, bool gring)
{
    const int64_t lim = cap - base;
    const uint32_t m = (int64_t)total < lim ? total : (lim > 0 ? (uint32_t)lim : 0u);
    T *d = dst + base;
    uint32_t j0 = 0;
    if (sizeof(T) >= 4) {
        // 16-byte loads from the (16-byte aligned) ring block, U in flight per lane:
        // the ring is read from L2 (~0.5-1 us per round trip) and phase stamps showed
        // the scalar copy (8 loads in flight) taking 5.4 us per 6 KB C2 block, which
        // backed up the compute warps' ring reservations.  Destination offsets are
        // arbitrary, so the stores stay element-wide.
        constexpr int V = 16 / sizeof(T);
        constexpr int U = 4;
        const uint4 *s4 = (const uint4 *)src;
        const uint32_t nv = m / V;
        uint32_t j = q;
        for (; j + (U - 1) * nq < nv; j += U * nq) {
            uint4 v[U];
#pragma unroll
            for (int u = 0; u < U; u++)
                v[u] = ld_ring(s4 + j + u * nq, gring);
#pragma unroll
            for (int u = 0; u < U; u++) {
                const T *e = (const T *)&v[u];
#pragma unroll
                for (int x = 0; x < V; x++)
                    d[(size_t)(j + u * nq) * V + x] = e[x];
            }
        }
        for (; j < nv; j += nq) {
            const uint4 v = ld_ring(s4 + j, gring);
            const T *e = (const T *)&v;
#pragma unroll
            for (int x = 0; x < V; x++)
                d[(size_t)j * V + x] = e[x];
        }
        j0 = nv * V;
    }
    // byte columns, and the last partial vector
    constexpr int U = 8;
    uint32_t j = j0 + q;
    for (; j + (U - 1) * nq < m; j += U * nq) {
        T v[U];
#pragma unroll
        for (int u = 0; u < U; u++)
            v[u] = ld_ring(src + j + u * nq, gring);
#pragma unroll
        for (int u = 0; u < U; u++)
            d[j + u * nq] = v[u];
    }
    for (; j < m; j += nq)
        d[j] = ld_ring(src + j, gring);
}

// Join expansion into a tile (§8(a) a8): candidates [t*T, t*T + rows) of the
// join output are mapped to (left row, right row) through the tile's run records
// (cached in smem) and the live join columns are gathered into the tile's slots.
// Thread `tid` expands candidates [tid*ITEMS, tid*ITEMS + ITEMS): one binary search,
// then a forward walk; ITEMS odd makes the thread-contiguous smem writes conflict-free.
template <int NT, int ITEMS>
__device__ inline void join_fill(const ChainProg &P, const JoinExpand &X, int64_t t, int64_t ntiles, int rows,
                                 char *st, char *rcache, const TileLaunch &L)
{
    constexpr int T = NT * ITEMS;
    const int tid = threadIdx.x;
    uint64_t *c_off = (uint64_t *)rcache;
    uint32_t *c_s = (uint32_t *)(c_off + (T + 1));
    uint32_t *c_lo = c_s + (T + 1);
    uint32_t *c_lenR = c_lo + (T + 1);
    const int64_t o0 = t * T;
    const int64_t r0 = X.tile_run[t];
    const int64_t r1 = (t + 1 < ntiles) ? X.tile_run[t + 1] : X.nruns - 1;
    const int nr = (int)(r1 - r0 + 1);
    for (int q = tid; q < nr; q += NT) {
        cp_async8(c_off + q, X.off + r0 + q);
        cp_async4(c_s + q, X.s + r0 + q);
        cp_async4(c_lo + q, X.lo + r0 + q);
        cp_async4(c_lenR + q, X.lenR + r0 + q);
    }
    cp_async_wait_all();
    bar_sync(kComputeBar, NT);
    if ((L.dbg & 4) && tid == 0)
        L.dbg_ts[12 * t + 10] = globaltimer();
    const int first = tid * ITEMS;
    if (first < rows) {
        uint32_t ii[ITEMS], jj[ITEMS];
        const uint64_t o = (uint64_t)(o0 + first);
        int lo = 0, hi = nr;
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (c_off[mid] <= o) lo = mid + 1;
            else hi = mid;
        }
        int r = lo - 1;
        // (i, j) of the first candidate by division, the rest by a carry walk: every
        // run has >= 1 candidate, so a step that leaves run r lands on the first
        // candidate (0, 0) of run r + 1
        const uint64_t d = o - c_off[r];
        uint32_t lr = c_lenR[r];
        uint32_t qi, qj;
        if (d == 0) {
            qi = qj = 0;
        } else if (d <= 0xffffffffull) {
            qi = (uint32_t)d / lr;
            qj = (uint32_t)d - qi * lr;
        } else {
            qi = (uint32_t)(d / lr);
            qj = (uint32_t)(d - (uint64_t)qi * lr);
        }
#pragma unroll
        for (int k = 0; k < ITEMS; k++) {
            ii[k] = jj[k] = 0;
            if (first + k < rows) {
                const uint64_t oo = o + k;
                if (r + 1 < nr && c_off[r + 1] <= oo) {
                    r++;
                    lr = c_lenR[r];
                    qi = qj = 0;
                }
                ii[k] = c_s[r] + qi;
                jj[k] = c_lo[r] + qj;
                if (++qj == lr) {
                    qj = 0;
                    ++qi;
                }
            }
        }
        // every gather of every live column is issued as an async copy before any
        // completes (one round trip per tile instead of one per column)
        for (int c = 0; c < X.ncols; c++) {
            char *dst = st + P.slot[X.dst_slot[c]].off;
            const int w = type_width(P.slot[X.dst_slot[c]].type);
            const char *src = (const char *)X.src[c];
            const bool right = X.from_right[c];
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                if (first + k < rows) {
                    const size_t row = right ? jj[k] : ii[k];
                    if (w == 4)
                        cp_async4((uint32_t *)dst + first + k, (const uint32_t *)src + row);
                    else if (w == 8)
                        cp_async8((uint64_t *)dst + first + k, (const uint64_t *)src + row);
                    else
                        ((uint8_t *)dst)[first + k] = ((const uint8_t *)src)[row];
                }
            }
        }
        cp_async_wait_all();
    }
    if ((L.dbg & 4) && tid == 0)
        L.dbg_ts[12 * t + 11] = globaltimer();
    bar_sync(kComputeBar, NT);
}

template <int NT, int ITEMS, bool AGG, bool JOIN, bool MULTI = false>
__global__ void __launch_bounds__(NT + aux_threads(AGG), AGG ? 1 : 2) k_scan_chain(const __grid_constant__ ChainProg P,
                                                                     const __grid_constant__ TileLaunch L,
                                                                     const __grid_constant__ JoinExpand X)
{
    constexpr int T = NT * ITEMS;
    constexpr int NW = NT / 32;             // compute warps
    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int S = L.stages;
    const uint32_t R = L.out_bytes;      // ring bytes (multiple of 128)
    ScanCtl<NT, ITEMS> *ctl = (ScanCtl<NT, ITEMS> *)smem_raw;
    char *stages = (char *)smem_raw + align_up(sizeof(ScanCtl<NT, ITEMS>), 128);
    char *scratch = stages + (size_t)S * P.stage_bytes;
    // compacted-tile ring: in smem, or (L.gring) a per-CTA slice of an L2-resident
    // global buffer, which leaves the shared memory to more input stages
    char *sm_ring = scratch + P.scratch_bytes;
    const bool gring = L.gring != nullptr;
    char *ring = gring ? L.gring + (size_t)blockIdx.x * R : sm_ring;
    char *sm_after = sm_ring + ((AGG || gring) ? 0 : R);
    unsigned long long *part = (unsigned long long *)sm_after;
    const int NA = P.nagg + 1;
    // agg_mode 0: thread-private int64 partials (D*NA*NT words); 2: partials in
    // registers (stored into the stage buffers at the end); then the CTA's 128-bit
    // accumulators
    const size_t part_words = AGG ? (P.agg_mode == 0 ? (size_t)P.D * NA * NT : 0) : 0;
    unsigned long long *cta_acc = part + part_words;
    char *rcache = sm_after;                // join: run-record cache for the current tile
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t n = L.n_ptr ? *L.n_ptr : L.n;
    const int64_t ntiles = (n + T - 1) / T;
    const bool emit = !AGG && !(L.dbg & 2) && !L.direct;
    // input-dependence branches: only the MULTI instance carries the branch loop, so
    // the single-chain instances compile with NB == 1
    const int NB = (AGG || JOIN || !MULTI) ? 1 : P.nbranch;

    if (tid == 0) {
        for (int s = 0; s < S; s++) {
            mbar_init(&ctl->in[s].full, 1);
            mbar_init(&ctl->in[s].empty, NW);          // one arrival per compute warp
        }
        for (int j = 0; j < kRingSlots; j++) {
            mbar_init(&ctl->blk[j].aggr, NW);          // one arrival per compute warp
            mbar_init(&ctl->blk[j].oempty, 1);
        }
        ctl->tail = 0;
        ctl->head = 0;
        ctl->hpos = 0;
        fence_mbar_init();
    }
    if constexpr (AGG) {
        for (size_t q = tid; q < part_words; q += blockDim.x)
            part[q] = 0;
        for (int q = tid; q < P.D * NA * 2; q += blockDim.x)
            cta_acc[q] = 0;
    }
    __syncthreads();

    constexpr int WW = AGG ? 0 : kWriterWarps;   // writer warps of this instance
    if (warp == NW + WW) {
        // ---------------- producer warp ----------------
        if (lane == 0) {
            uint32_t tx_bytes = 0;
            for (int i = 0; i < P.nin; i++)
                tx_bytes += (uint32_t)T * type_width(P.slot[i].type);
            const uint64_t policy = policy_evict_first();
            int s = 0;
            uint32_t eph = 1;                                // parity of the previous use
            for (int64_t i = 0;; ++i) {
                if (i >= S)
                    mbar_wait_aux(&ctl->in[s].empty, eph, 64, L.dbg);
                const int64_t t = (int64_t)atomicAdd(&L.ctrs[0], 1u);
                ctl->in[s].tile = t;
                if ((L.dbg & 4) && t < ntiles)
                    L.dbg_ts[12 * t + 0] = globaltimer();
                if (!JOIN && t < ntiles && L.use_tma && (t + 1) * (int64_t)T <= n) {
                    char *st = stages + (size_t)s * P.stage_bytes;
                    fence_proxy_async_smem();
                    mbar_arrive_expect_tx(&ctl->in[s].full, tx_bytes);
                    for (int c = 0; c < P.nin; c++) {
                        const int w = type_width(P.slot[c].type);
                        bulk_g2s(st + P.slot[c].off, (const char *)P.in_ptr[c] + (size_t)t * T * w,
                                 (uint32_t)T * w, &ctl->in[s].full, policy);
                    }
                } else {
                    mbar_arrive(&ctl->in[s].full);
                }
                if (t >= ntiles)
                    break;
                if (++s == S) {
                    s = 0;
                    eph ^= 1;
                }
            }
        }
    } else if (warp >= NW) {
        // ---------------- writer warps: look-back + compacted store ----------------
        // Writer w owns ring slots i = w (mod kWriterWarps): the look-backs and copies
        // of consecutive tiles proceed concurrently; ring bytes are released in order.
        const int wi = warp - NW;
        if (emit) {
            for (int64_t i = wi;; i += kWriterWarps) {
                const int j = (int)(i % kRingSlots);
                mbar_wait_aux(&ctl->blk[j].aggr, (uint32_t)((i / kRingSlots) & 1), 256, L.dbg);
                const int64_t t = ctl->blk[j].tile;
                if (t >= ntiles)
                    break;
                const uint32_t total = ctl->blk[j].total;
                const int b = (int)ctl->blk[j].br;
                if ((L.dbg & 4) && lane == 0)
                    L.dbg_ts[12 * t + 5] = globaltimer();
                const int64_t excl = (L.dbg & 1) ? t * T
                                                  : (int64_t)lookback_warp(L.status + b * L.status_stride, t, total, L.epoch,
                                                                           /*aggregate_published=*/true,
                                                                           (L.dbg & 128) ? 0u : (L.dbg & 64) ? 256u : (L.dbg & 256) ? 4096u : 1024u);
                if (lane == 0) {
                    if (L.dbg & 4)
                        L.dbg_ts[12 * t + 3] = globaltimer();
                    if (t == ntiles - 1)
                        *(b ? L.br_n_dev[b] : L.n_dev) = excl + (int64_t)total;
                }
                const char *blk = ring + ctl->blk[j].roff;
                const int64_t cap = b ? P.br_cap[b] : P.out_capacity;
                uint32_t coff = 0;
                for (int c = b ? P.br_out_end[b - 1] : 0; c < (NB > 1 ? (int)P.br_out_end[b] : P.nout); c++) {
                    const int w = P.out_w[c];
                    const char *src = blk + coff;
                    coff += al16(total * w);
                    switch (w) {
                    case 1: group_copy_out<uint8_t>((uint8_t *)P.out_ptr[c], (const uint8_t *)src, excl, total, cap, lane, 32, gring); break;
                    case 4: group_copy_out<uint32_t>((uint32_t *)P.out_ptr[c], (const uint32_t *)src, excl, total, cap, lane, 32, gring); break;
                    default: group_copy_out<uint64_t>((uint64_t *)P.out_ptr[c], (const uint64_t *)src, excl, total, cap, lane, 32, gring); break;
                    }
                }
                __syncwarp();
                if (gring && !(L.dbg & 8)) {
                    // the block has been copied out (every loaded value was stored): drop
                    // its fully covered L2 lines so the ring never costs DRAM write-back
                    const uintptr_t b0 = ((uintptr_t)blk + 127) & ~(uintptr_t)127;
                    const uintptr_t b1 = ((uintptr_t)blk + coff) & ~(uintptr_t)127;
                    for (uintptr_t a = b0 + (uintptr_t)lane * 128; a < b1; a += 32 * 128)
                        discard_l2_line((const void *)a);
                    __syncwarp();
                }
                if (lane == 0) {
                    if (L.dbg & 4)
                        L.dbg_ts[12 * t + 4] = globaltimer();
                    if (i > 0)   // release ring bytes in tile order
                        mbar_wait_aux(&ctl->blk[(i - 1) % kRingSlots].oempty, (uint32_t)(((i - 1) / kRingSlots) & 1), 64, L.dbg);
                    // the discards must land in L2 before the bytes can be rewritten
                    if (gring && !(L.dbg & 8))
                        __threadfence();
                    else
                        __threadfence_block();
                    ctl->tail = ctl->tail + ctl->blk[j].used;
                    mbar_arrive(&ctl->blk[j].oempty);
                }
                __syncwarp();
            }
        }
    } else {
        // ---------------- compute warps ----------------
        // Every thread reads and writes only its own rows (k*NT + tid) of the stage and
        // of the scratch tile, so warps run independently: the only CTA-wide barrier per
        // tile is the one that makes the survivor counts visible.  The stage is released
        // and the compacted block handed to the writers by per-warp mbarrier arrivals
        // (count = NW); the ring reservation is replicated, deterministically, in every warp.
        int64_t since_flush = 0;
        RegAgg racc;
        if (AGG && P.agg_mode == 2)
            reg_agg_zero(racc);
        int s = 0;
        uint32_t fph = 0;
        uint32_t head = 0, hpos = 0;
        int64_t ublk = 0;                                 // compacted blocks emitted (tiles x branches)
        for (int64_t i = 0;; ++i) {
            if (i > 0 && ++s == S) {
                s = 0;
                fph ^= 1;
            }
            mbar_wait(&ctl->in[s].full, fph);
            const int64_t t = ctl->in[s].tile;
            if (t >= ntiles) {
                if (emit && tid == 0) {
                    // one sentinel per writer warp (consecutive slots)
                    for (int64_t u = ublk; u < ublk + kWriterWarps; ++u) {
                        const int ju = (int)(u % kRingSlots);
                        if (u >= kRingSlots)
                            mbar_wait(&ctl->blk[ju].oempty, (uint32_t)(((u / kRingSlots) - 1) & 1));
                        ctl->blk[ju].tile = ntiles;
                        mbar_arrive_cnt(&ctl->blk[ju].aggr, NW);
                    }
                }
                if (AGG && P.agg_mode == 2)
                    reg_agg_reduce_warp(P, racc, cta_acc);   // warp-reduced, 128-bit exact
                break;
            }
            char *st = stages + (size_t)s * P.stage_bytes;
            const int64_t row0 = t * T;
            const int rows = (int)min((int64_t)T, n - row0);
            if ((L.dbg & 4) && tid == 0)
                L.dbg_ts[12 * t + 1] = globaltimer();
            auto release_stage = [&]() {
                __syncwarp();
                if (lane == 0)
                    mbar_arrive(&ctl->in[s].empty);
            };
            if (L.dbg & 2) {   // diagnostics: stream the tiles only (TMA pipeline ceiling)
                release_stage();
                continue;
            }
            if (JOIN) {
                join_fill<NT, ITEMS>(P, X, t, ntiles, rows, st, rcache, L);
            } else if (!(L.use_tma && rows == T)) {
                // ragged last tile or unaligned column bases: each thread loads its own rows
                for (int c = 0; c < P.nin; c++) {
                    const int w = type_width(P.slot[c].type);
                    char *dst = st + P.slot[c].off;
                    const char *src = (const char *)P.in_ptr[c] + (size_t)row0 * w;
                    if (w == 4) {
                        for (int r = tid; r < rows; r += NT)
                            ((uint32_t *)dst)[r] = ((const uint32_t *)src)[r];
                    } else if (w == 8) {
                        for (int r = tid; r < rows; r += NT)
                            ((uint64_t *)dst)[r] = ((const uint64_t *)src)[r];
                    } else {
                        for (int r = tid; r < rows; r += NT)
                            dst[r] = src[r];
                    }
                }
            }
            uint32_t mask0 = (1u << ITEMS) - 1u;
            if (rows < T) {
                mask0 = 0;
#pragma unroll
                for (int k = 0; k < ITEMS; k++)
                    if (k * NT + tid < rows)
                        mask0 |= 1u << k;
            }
            uint32_t mask = run_ops<NT, ITEMS>(P, 0, NB > 1 ? (int)P.br_op_end[0] : P.nops, st, scratch, mask0);
            if ((L.dbg & 4) && tid == 0)
                L.dbg_ts[12 * t + 6] = globaltimer();
            if (AGG) {
                if (P.agg_mode == 2)
                    agg_tile_reg<NT, ITEMS>(P, st, scratch, mask, racc, cta_acc, since_flush, L.err);
                else if (P.agg_mode == 3)
                    agg_tile_global<NT, ITEMS>(P, st, scratch, mask, L.agg_acc, L.err);
                else
                    agg_tile<NT, ITEMS>(P, st, scratch, mask, part, cta_acc, since_flush, L.err);
                if ((L.dbg & 4) && tid == 0)
                    L.dbg_ts[12 * t + 2] = globaltimer();
                release_stage();
                continue;
            }
            if (L.direct) {
                // every row survives: coalesced stores at the rows' own offsets
                const int64_t lim64 = min((int64_t)rows, P.out_capacity - row0);
                const int lim = (int)(lim64 > 0 ? lim64 : 0);
                for (int c = 0; c < P.nout; c++) {
                    const char *src = loc_ptr(P.out_loc[c], st, scratch);
                    switch (P.out_w[c]) {
                    case 1:
#pragma unroll
                        for (int k = 0; k < ITEMS; k++)
                            if (k * NT + tid < lim) ((uint8_t *)P.out_ptr[c])[row0 + k * NT + tid] = ((const uint8_t *)src)[k * NT + tid];
                        break;
                    case 4:
#pragma unroll
                        for (int k = 0; k < ITEMS; k++)
                            if (k * NT + tid < lim) ((uint32_t *)P.out_ptr[c])[row0 + k * NT + tid] = ((const uint32_t *)src)[k * NT + tid];
                        break;
                    default:
#pragma unroll
                        for (int k = 0; k < ITEMS; k++)
                            if (k * NT + tid < lim) ((uint64_t *)P.out_ptr[c])[row0 + k * NT + tid] = ((const uint64_t *)src)[k * NT + tid];
                        break;
                    }
                }
                release_stage();
                continue;
            }
            // one compacted block per branch (input-dependence fusion, §4.4): the
            // branches share the staged tile and differ in their ops, mask and outputs
            for (int b = 0;; ) {
                const int j = (int)(ublk % kRingSlots);
                uint32_t *cnt = ctl->cnt[ublk & 1];
                uint32_t bal[ITEMS];
#pragma unroll
                for (int k = 0; k < ITEMS; k++) {
                    bal[k] = __ballot_sync(0xffffffffu, (mask >> k) & 1u);
                    if (lane == 0)
                        cnt[k * NW + warp] = __popc(bal[k]);
                }
                bar_sync(kComputeBar, NT);
                if ((L.dbg & 4) && tid == 0)
                    L.dbg_ts[12 * t + 7] = globaltimer();
                // every warp scans the ITEMS x NW survivor counts itself
                uint32_t pre[ITEMS];
                uint32_t total;
                {
                    constexpr int NV = ITEMS * NW;
                    constexpr int PER = (NV + 31) / 32;
                    uint32_t v[PER];
                    uint32_t sum = 0;
#pragma unroll
                    for (int qq = 0; qq < PER; qq++) {
                        const int idx = lane * PER + qq;
                        v[qq] = idx < NV ? cnt[idx] : 0;
                        sum += v[qq];
                    }
                    uint32_t inc = sum;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
                        if (lane >= o)
                            inc += y;
                    }
                    total = __shfl_sync(0xffffffffu, inc, 31);
                    const uint32_t base = inc - sum;
#pragma unroll
                    for (int k = 0; k < ITEMS; k++) {
                        const int idx = k * NW + warp;
                        const int owner = idx / PER, off = idx % PER;
                        uint32_t part_sum = 0;
#pragma unroll
                        for (int qq = 0; qq < PER; qq++)
                            if (qq < off) part_sum += v[qq];
                        pre[k] = __shfl_sync(0xffffffffu, base + part_sum, owner);
                    }
                }
                if (warp == 0 && lane == 31) {
                    // publish the tile aggregate before anything can block this CTA
                    if (t > 0 && !(L.dbg & 1))
                        st_relaxed_u64(&L.status[b * L.status_stride + t], ((uint64_t)L.epoch << 48) | (1ull << 46) | total);
                    if (L.dbg & 4)
                        L.dbg_ts[12 * t + 2] = globaltimer();
                }
                // ring bytes for the compacted tile (blocks never wrap); every warp computes
                // the same reservation from the same (head, hpos, total)
                const int c0 = b ? P.br_out_end[b - 1] : 0, c1 = NB > 1 ? (int)P.br_out_end[b] : P.nout;
                uint32_t need = 0;
                for (int c = c0; c < c1; c++)
                    need += al16(total * P.out_w[c]);
                if ((L.dbg & 4) && tid == 0)
                    L.dbg_ts[12 * t + 9] = globaltimer();
                uint32_t pos = hpos;
                uint32_t used = need;
                bool drain = false;
                if (pos + need > R) {           // skip the tail [pos, R)
                    used += R - pos;
                    pos = 0;
                    if (used > R) {             // cannot fit behind live blocks: wait for an empty ring
                        used = need;
                        drain = true;
                    }
                }
                if (ublk >= kRingSlots)
                    mbar_wait(&ctl->blk[j].oempty, (uint32_t)(((ublk / kRingSlots) - 1) & 1));
                {
                    uint32_t backoff = 32;
                    while (drain ? (head != ctl->tail) : (head + used - ctl->tail > R)) {
                        __nanosleep(backoff);
                        backoff = backoff < 512 ? backoff * 2 : 512;
                    }
                }
                head += used;
                hpos = pos + need == R ? 0 : pos + need;
                char *blk = ring + pos;
                const uint32_t lt = lanemask_lt();
                uint32_t posk[ITEMS];
#pragma unroll
                for (int k = 0; k < ITEMS; k++)
                    posk[k] = pre[k] + __popc(bal[k] & lt);
                uint32_t coff = 0;
                for (int c = c0; c < c1 && !(L.dbg & 1024); c++) {   // dbg 1024: skip the ring stores (ablation)
                    const int w = P.out_w[c];
                    const char *src = loc_ptr(P.out_loc[c], st, scratch);
                    char *dst = blk + coff;
                    coff += al16(total * w);
                    switch (w) {
                    case 1:
#pragma unroll
                        for (int k = 0; k < ITEMS; k++)
                            if ((mask >> k) & 1u) ((uint8_t *)dst)[posk[k]] = ((const uint8_t *)src)[k * NT + tid];
                        break;
                    case 4:
#pragma unroll
                        for (int k = 0; k < ITEMS; k++)
                            if ((mask >> k) & 1u) ((uint32_t *)dst)[posk[k]] = ((const uint32_t *)src)[k * NT + tid];
                        break;
                    default:
#pragma unroll
                        for (int k = 0; k < ITEMS; k++)
                            if ((mask >> k) & 1u) ((uint64_t *)dst)[posk[k]] = ((const uint64_t *)src)[k * NT + tid];
                        break;
                    }
                }
                __syncwarp();
                if (lane == 0) {
                    if (gring && !(L.dbg & 512))
                        __threadfence_block();
                    if (warp == 0) {
                        ctl->blk[j].tile = t;
                        ctl->blk[j].total = total;
                        ctl->blk[j].roff = pos;
                        ctl->blk[j].used = used;
                        ctl->blk[j].br = (uint32_t)b;
                    }
                    if (b == NB - 1)
                        mbar_arrive(&ctl->in[s].empty);      // this warp is done with the stage
                    mbar_arrive(&ctl->blk[j].aggr);          // and with the ring block
                    if ((L.dbg & 4) && warp == 0)
                        L.dbg_ts[12 * t + 8] = globaltimer();
                }
                ++ublk;
                if (++b == NB)
                    break;
                mask = run_ops<NT, ITEMS>(P, P.br_op_end[b - 1], P.br_op_end[b], st, scratch, mask0);
            }
        }
    }
    __syncthreads();
    if (AGG) {
        if (P.agg_mode == 0)      // modes 2 / 3 added their rows into cta_acc / the global accumulators already
            agg_combine<NT>(P, part, cta_acc, blockDim.x);
        __syncthreads();
        for (int qq = tid; qq < P.D * NA; qq += blockDim.x) {
            const unsigned long long lo = cta_acc[2 * qq], hi = cta_acc[2 * qq + 1];
            if (lo | hi)
                atomic_add128(&L.agg_acc[2 * qq], &L.agg_acc[2 * qq + 1], lo, hi);
        }
    } else if ((ntiles == 0 || L.direct) && blockIdx.x == 0 && tid == 0) {
        *L.n_dev = L.direct ? n : 0;
        for (int b = 1; b < NB; b++)
            *L.br_n_dev[b] = 0;
    }
    cta_exit_reset(L.ctrs);
}

// ===========================================================================
// Aggregate finalisation: one CTA scans the D groups, emits those with count>0
// in ascending code order (reading A12), and zeroes the accumulators.
// ===========================================================================
__global__ void __launch_bounds__(kThreads) k_agg_finalize(const __grid_constant__ AggFinal F)
{
    __shared__ uint32_t wsum[kWarps];
    __shared__ int64_t base;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0)
        base = 0;
    __syncthreads();
    for (int g0 = 0; g0 < F.D; g0 += kThreads) {
        const int g = g0 + tid;
        unsigned long long cnt = 0;
        if (g < F.D)
            cnt = F.acc[2 * ((size_t)g * F.NA)];
        const bool live = cnt > 0;
        uint32_t b = __ballot_sync(0xffffffffu, live);
        if (lane == 0)
            wsum[warp] = __popc(b);
        __syncthreads();
        uint32_t before = 0, total = 0;
        for (int w = 0; w < kWarps; w++) {
            if (w < warp)
                before += wsum[w];
            total += wsum[w];
        }
        const int64_t pos = base + before + __popc(b & lanemask_lt());
        if (live && pos < F.capacity) {
            int oc = 0;
            int rem = g;
            int codes[kMaxGroupCols];
            for (int c = F.ngc - 1; c >= 0; c--) {
                codes[c] = rem % F.gdomain[c];
                rem /= F.gdomain[c];
            }
            for (int c = 0; c < F.ngc; c++, oc++) {
                switch (type_width(F.gtype[c])) {
                case 1: ((uint8_t *)F.out[oc])[pos] = (uint8_t)codes[c]; break;
                case 4: ((uint32_t *)F.out[oc])[pos] = (uint32_t)codes[c]; break;
                default: ((uint64_t *)F.out[oc])[pos] = (uint64_t)codes[c]; break;
                }
            }
            for (int q = 0; q < F.nreq; q++) {
                const size_t a = (size_t)g * F.NA + F.req_acc[q];
                if (F.req_is_sum[q]) {
                    ((unsigned long long *)F.out[oc++])[pos] = F.acc[2 * a];
                    ((unsigned long long *)F.out[oc++])[pos] = F.acc[2 * a + 1];
                } else {
                    ((unsigned long long *)F.out[oc++])[pos] = F.acc[2 * a];
                }
            }
        }
        __syncthreads();
        if (g < F.D)
            for (int a = 0; a < F.NA; a++) {
                F.acc_w[2 * ((size_t)g * F.NA + a)] = 0;
                F.acc_w[2 * ((size_t)g * F.NA + a) + 1] = 0;
            }
        if (tid == 0)
            base += total;
        __syncthreads();
    }
    if (tid == 0) {
        *F.n_dev = base;
        F.err[1] = F.err[0];
        F.err[0] = 0;
        F.err[3] = F.err[2];
        F.err[2] = 0;
    }
}

// ===========================================================================
// JOIN phase 1 — merge-path partitions of the merged key sequence (L before R on
// ties, §4.3.2 binary-search partitioning).  For every L element that
// starts a key run inside the partition: R range [lo, hi) by binary search in
// the partition's smem copy of R (lo always lies inside it), galloping past the
// partition end for long runs; L run length likewise.  Runs with a match are
// compacted (ballot + look-back) into run records with their output offsets.
// ===========================================================================
constexpr int kRunItems = 8;
constexpr int kRunT = kThreads * kRunItems;
constexpr int kRunExt = 512;     // extra L / R elements staged past the partition end

template <typename K>
__device__ __forceinline__ int64_t merge_path(const K *L, int64_t nl, const K *R, int64_t nr, int64_t d)
{
    int64_t lo = d > nr ? d - nr : 0;
    int64_t hi = d < nl ? d : nl;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (L[mid] <= R[d - mid - 1])
            lo = mid + 1;
        else
            hi = mid;
    }
    return lo;
}

template <typename K>
__device__ __forceinline__ int lower_bound_smem(const K *a, int n, K key)
{
    int lo = 0, hi = n;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (a[mid] < key) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

template <typename K>
__device__ __forceinline__ int upper_bound_smem(const K *a, int n, K key)
{
    int lo = 0, hi = n;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (a[mid] <= key) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// first index >= start with A[idx] > key (A[start..] sorted, A[start-1] <= key)
template <typename K>
__device__ int64_t gallop_upper(const K *A, int64_t start, int64_t n, K key)
{
    int64_t lo = start, hi = n, step = 1;
    while (true) {
        int64_t probe = lo + step - 1;
        if (probe >= n) { hi = n; break; }
        if (A[probe] > key) { hi = probe; break; }
        lo = probe + 1;
        step <<= 1;
    }
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (A[mid] <= key) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// exclusive block scan of per-(item, thread) 64-bit values in (k, warp, lane) order
template <int ITEMS>
__device__ inline void block_scan_u64(uint64_t (&v)[ITEMS], uint64_t *wtot /* ITEMS*kWarps */, uint64_t &total)
{
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        uint64_t x = v[k], inc = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o)
                inc += y;
        }
        v[k] = inc - x;   // exclusive within the warp
        if (lane == 31)
            wtot[k * kWarps + warp] = inc;
    }
    __syncthreads();
    if (warp == 0) {
        constexpr int NV = ITEMS * kWarps;
        constexpr int PER = (NV + 31) / 32;
        uint64_t a[PER];
        uint64_t s = 0;
#pragma unroll
        for (int q = 0; q < PER; q++) {
            int idx = lane * PER + q;
            a[q] = idx < NV ? wtot[idx] : 0;
            s += a[q];
        }
        uint64_t inc = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint64_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o)
                inc += y;
        }
        uint64_t run = inc - s;
#pragma unroll
        for (int q = 0; q < PER; q++) {
            int idx = lane * PER + q;
            if (idx < NV)
                wtot[idx] = run;
            run += a[q];
        }
        if (lane == 31)
            wtot[NV] = inc;
    }
    __syncthreads();
    total = wtot[ITEMS * kWarps];
#pragma unroll
    for (int k = 0; k < ITEMS; k++)
        v[k] += wtot[k * kWarps + warp];
}

// merge-path split of every partition boundary d = p * kRunT (p = 0..nparts)
template <typename K>
__global__ void k_merge_splits(const __grid_constant__ JoinRunsLaunch J)
{
    const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (p > J.nparts)
        return;
    const int64_t d = min(p * kRunT, J.nl + J.nr);
    J.split[p] = merge_path((const K *)J.lkey, J.nl, (const K *)J.rkey, J.nr, d);
}

// first index in [start, n) of a sorted smem array with a[idx] > key (a[start-1] <= key)
template <typename K>
__device__ __forceinline__ int gallop_smem(const K *a, int start, int n, K key)
{
    int lo = start, hi = n, step = 1;
    while (true) {
        const int probe = lo + step - 1;
        if (probe >= n) { hi = n; break; }
        if (a[probe] > key) { hi = probe; break; }
        lo = probe + 1;
        step <<= 1;
    }
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (a[mid] <= key) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// fused upstream SELECT on the join key (N2): every atom must hold for the run's key
template <typename K>
__device__ __forceinline__ bool key_pass(const JoinRunsLaunch &J, K key)
{
    bool ok = true;
    for (int i = 0; i < J.nkpred; i++) {
        const K c = (K)J.kpk[i];
        switch (J.kop[i]) {
        case C_LT: ok = ok && key < c; break;
        case C_LE: ok = ok && key <= c; break;
        case C_GT: ok = ok && key > c; break;
        case C_GE: ok = ok && key >= c; break;
        case C_EQ: ok = ok && key == c; break;
        default: ok = ok && key != c; break;
        }
    }
    return ok;
}

// Two streaming passes (no look-back on the critical path): WRITE = false counts
// the matched runs and join candidates of every partition; k_scan_parts turns the
// counts into exclusive offsets; WRITE = true recomputes the partition (identical
// arithmetic) and writes the run records at their offsets.
//
// In the merged order (L before R on equal keys, P:196 binary-search partitioning)
// every key forms one contiguous segment [its L rows][its R rows].  A segment HEAD is
// a merged element whose key differs from its predecessor's; at a head the walk's
// (L index, R index) are the key's first L row and its R lower bound, and the next
// head's indices end both runs.  So a partition needs no per-run searches:
//   1. each thread merges its 8 positions (one diagonal search) and records heads;
//   2. a block scan places the heads in smem in merged order;
//   3. head k's run lengths are head k+1's indices minus its own; only the
//      partition's last head looks past the partition end (galloping in smem, then
//      in HBM for hot keys whose segment spans later partitions);
//   4. matched heads (lenL > 0 and lenR > 0) are compacted into run records.
template <typename K, bool WRITE>
__global__ void __launch_bounds__(kThreads, 3) k_join_runs(const __grid_constant__ JoinRunsLaunch J)
{
    extern __shared__ __align__(128) unsigned char smem_raw[];
    uint64_t *wtot = (uint64_t *)smem_raw;                        // 2 * kWarps, then head counts
    int32_t *hcount = (int32_t *)(wtot + 2 * kWarps);             // kWarps
    K *sL = (K *)(smem_raw + align_up((kRunItems * kWarps + 1) * 8, 128));   // kRunT + kRunExt
    K *sR = sL + kRunT + kRunExt;                                 // kRunT + kRunExt
    int32_t *hL = (int32_t *)(sR + kRunT + kRunExt);              // kRunT heads (local L index)
    int32_t *hR = hL + kRunT;                                     // kRunT heads (local R index)
    K *hK = (K *)align_up((size_t)(hR + kRunT), 16);              // kRunT head keys
    const K *L = (const K *)J.lkey;
    const K *R = (const K *)J.rkey;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t ntot = J.nl + J.nr;

    // software pipeline: the keys of the CTA's next partition are loaded into
    // registers while the current one is processed
    constexpr int PF = (kRunT + kRunExt + kThreads - 1) / kThreads;
    K pfL[PF], pfR[PF];
    auto fetch = [&](int64_t pp) {
        const int64_t a0 = J.split[pp], a1 = J.split[pp + 1];
        const int64_t e0 = min(pp * kRunT, ntot);
        const int64_t b0 = e0 - a0, b1 = min(e0 + kRunT, ntot) - a1;
        const int nle = (int)(min(a1 + kRunExt, J.nl) - a0), nre = (int)(min(b1 + kRunExt, J.nr) - b0);
#pragma unroll
        for (int q = 0; q < PF; q++) {
            const int idx = tid + q * kThreads;
            pfL[q] = idx < nle ? L[a0 + idx] : K(0);
            pfR[q] = idx < nre ? R[b0 + idx] : K(0);
        }
    };
    if ((int64_t)blockIdx.x < J.nparts)
        fetch(blockIdx.x);
    for (int64_t p = blockIdx.x; p < J.nparts; p += gridDim.x) {
        const int64_t d0 = p * kRunT, d1 = min(d0 + kRunT, ntot);
        const int64_t i0 = J.split[p], i1 = J.split[p + 1], j0 = d0 - i0, j1 = d1 - i1;
        const int nL = (int)(i1 - i0), nR = (int)(j1 - j0), m = (int)(d1 - d0);
        const int nLe = (int)(min(i1 + kRunExt, J.nl) - i0), nRe = (int)(min(j1 + kRunExt, J.nr) - j0);
        __syncthreads();
#pragma unroll
        for (int q = 0; q < PF; q++) {
            const int idx = tid + q * kThreads;
            if (idx < nLe) sL[idx] = pfL[q];
            if (idx < nRe) sR[idx] = pfR[q];
        }
        __syncthreads();
        if (p + gridDim.x < J.nparts)
            fetch(p + gridDim.x);

        // 1. merge walk over the thread's positions: bit q of hmask = position dt+q is a
        //    segment head, bit q of tmask = it is an L element (so its L index is lo0 +
        //    popc(tmask below q) and its R index the merged position minus that)
        uint32_t hmask = 0, tmask = 0;
        int lo0 = 0;
        const int dt = tid * kRunItems;
        if (dt < m) {
            int lo = dt > nR ? dt - nR : 0, hi = dt < nL ? dt : nL;
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if (sL[mid] <= sR[dt - mid - 1]) lo = mid + 1;
                else hi = mid;
            }
            lo0 = lo;
            int li = lo, rj = dt - lo;
            // predecessor of the first position in merged order: the larger of the
            // preceding L and R elements (global ones at the partition start)
            const bool pl_ok = (i0 + li) > 0, pr_ok = (j0 + rj) > 0;
            bool has_prev = pl_ok || pr_ok;
            K prev = K(0);
            if (has_prev) {
                const K pl = pl_ok ? (li > 0 ? sL[li - 1] : L[i0 - 1]) : K(0);
                const K pr = pr_ok ? (rj > 0 ? sR[rj - 1] : R[j0 - 1]) : K(0);
                prev = !pl_ok ? pr : (!pr_ok ? pl : (pl < pr ? pr : pl));
            }
#pragma unroll
            for (int q = 0; q < kRunItems; q++) {
                if (dt + q < m) {
                    const bool takeL = rj >= nR || (li < nL && sL[li] <= sR[rj]);
                    const K key = takeL ? sL[li] : sR[rj];
                    hmask |= (uint32_t)(!has_prev || key != prev) << q;
                    tmask |= (uint32_t)takeL << q;
                    has_prev = true;
                    prev = key;
                    li += takeL ? 1 : 0;
                    rj += takeL ? 0 : 1;
                }
            }
        }
        const int nh = __popc(hmask);
        // 2. heads in merged order into smem
        int hinc = nh;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, hinc, o);
            if (lane >= o) hinc += y;
        }
        if (lane == 31)
            hcount[warp] = hinc;
        __syncthreads();
        int hbase = 0, H = 0;
        for (int w = 0; w < kWarps; w++) {
            if (w < warp) hbase += hcount[w];
            H += hcount[w];
        }
        hbase += hinc - nh;
        for (uint32_t hm = hmask; hm; hm &= hm - 1) {
            const int q = __ffs(hm) - 1;
            const int li = lo0 + __popc(tmask & ((1u << q) - 1u));
            const int rj = dt + q - li;
            hL[hbase] = li;
            hR[hbase] = rj;
            hK[hbase] = ((tmask >> q) & 1u) ? sL[li] : sR[rj];
            hbase++;
        }
        __syncthreads();
        // 3. run lengths; the last head's segment may continue past the partition
        const int k0 = tid * kRunItems;
        int64_t tailL = 0, tailR = 0;
        if (k0 < H && k0 + kRunItems >= H) {
            const K key = hK[H - 1];
            int e = nL;
            if (nL < nLe && sL[nL] == key)
                e = gallop_smem(sL, nL + 1, nLe, key);
            tailL = i0 + e;
            if (e == nLe && i0 + e < J.nl && L[i0 + e] == key)
                tailL = gallop_upper(L, i0 + e, J.nl, key);
            int f = nR;
            if (nR < nRe && sR[nR] == key)
                f = gallop_smem(sR, nR + 1, nRe, key);
            tailR = j0 + f;
            if (f == nRe && j0 + f < J.nr && R[j0 + f] == key)
                tailR = gallop_upper(R, j0 + f, J.nr, key);
        }
        int nrun = 0;
        uint64_t outs = 0;
        uint32_t matched = 0;
        uint64_t cnt[kRunItems];
        int64_t lenl[kRunItems], lenr[kRunItems];
#pragma unroll
        for (int q = 0; q < kRunItems; q++) {
            const int k = k0 + q;
            cnt[q] = 0;
            lenl[q] = lenr[q] = 0;
            if (k < H) {
                const int64_t nl_ = k + 1 < H ? i0 + hL[k + 1] : tailL;
                const int64_t nr_ = k + 1 < H ? j0 + hR[k + 1] : tailR;
                lenl[q] = nl_ - (i0 + hL[k]);
                lenr[q] = nr_ - (j0 + hR[k]);
                if (lenl[q] > 0 && lenr[q] > 0 && key_pass<K>(J, hK[k])) {
                    matched |= 1u << q;
                    cnt[q] = (uint64_t)lenl[q] * (uint64_t)lenr[q];
                    nrun++;
                    outs += cnt[q];
                }
            }
        }
        // 4. block exclusive scan of (runs, outputs) over threads (thread order = merge order)
        uint64_t ir = (uint64_t)nrun, io = outs;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint64_t yr = __shfl_up_sync(0xffffffffu, ir, o), yo = __shfl_up_sync(0xffffffffu, io, o);
            if (lane >= o) {
                ir += yr;
                io += yo;
            }
        }
        if (lane == 31) {
            wtot[warp] = ir;
            wtot[kWarps + warp] = io;
        }
        __syncthreads();
        uint64_t br = 0, bo = 0, tr = 0, to = 0;
        for (int w = 0; w < kWarps; w++) {
            if (w < warp) {
                br += wtot[w];
                bo += wtot[kWarps + w];
            }
            tr += wtot[w];
            to += wtot[kWarps + w];
        }
        br += ir - (uint64_t)nrun;
        bo += io - outs;
        if (!WRITE) {
            if (tid == 0) {
                J.pruns[p] = tr;
                J.pouts[p] = to;
            }
            continue;
        }
        int64_t r = (int64_t)J.pruns[p] + (int64_t)br;
        uint64_t off = J.pouts[p] + bo;
#pragma unroll
        for (int q = 0; q < kRunItems; q++) {
            if ((matched >> q) & 1u) {
                const int k = k0 + q;
                if (r < J.cap_runs) {
                    J.s[r] = (uint32_t)(i0 + hL[k]);
                    J.lenL[r] = (uint32_t)lenl[q];
                    J.lo[r] = (uint32_t)(j0 + hR[k]);
                    J.lenR[r] = (uint32_t)lenr[q];
                    J.off[r] = off;
                }
                r++;
                off += cnt[q];
            }
        }
    }
}

// exclusive scan of the per-partition counts (one CTA; nparts is ~ rows / 2048)
__global__ void __launch_bounds__(1024) k_scan_parts(const __grid_constant__ JoinRunsLaunch J)
{
    __shared__ uint64_t wr[32], wo[32];
    __shared__ uint64_t carry_r, carry_o;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0)
        carry_r = carry_o = 0;
    __syncthreads();
    for (int64_t b0 = 0; b0 < J.nparts; b0 += 1024) {
        const int64_t p = b0 + tid;
        const uint64_t r = p < J.nparts ? J.pruns[p] : 0, o = p < J.nparts ? J.pouts[p] : 0;
        uint64_t ir = r, io = o;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint64_t yr = __shfl_up_sync(0xffffffffu, ir, d), yo = __shfl_up_sync(0xffffffffu, io, d);
            if (lane >= d) {
                ir += yr;
                io += yo;
            }
        }
        if (lane == 31) {
            wr[warp] = ir;
            wo[warp] = io;
        }
        __syncthreads();
        if (warp == 0) {
            uint64_t xr = wr[lane], xo = wo[lane];
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint64_t yr = __shfl_up_sync(0xffffffffu, xr, d), yo = __shfl_up_sync(0xffffffffu, xo, d);
                if (lane >= d) {
                    xr += yr;
                    xo += yo;
                }
            }
            wr[lane] = xr;
            wo[lane] = xo;
        }
        __syncthreads();
        const uint64_t er = carry_r + (warp ? wr[warp - 1] : 0) + ir - r;
        const uint64_t eo = carry_o + (warp ? wo[warp - 1] : 0) + io - o;
        if (p < J.nparts) {
            J.pruns[p] = er;
            J.pouts[p] = eo;
        }
        __syncthreads();
        if (tid == 0) {
            carry_r += wr[31];
            carry_o += wo[31];
        }
        __syncthreads();
    }
    if (tid == 0) {
        J.totals[0] = (int64_t)carry_r;
        J.totals[1] = (int64_t)carry_o;
    }
}

// first run of every expansion tile: tile_run[t] = upper_bound(off, t*T) - 1
__global__ void k_tile_runs(const uint64_t *off, int64_t nruns, int64_t ntiles, int64_t T, int64_t *tile_run)
{
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= ntiles)
        return;
    const uint64_t o = (uint64_t)(t * T);
    int64_t lo = 0, hi = nruns;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (off[mid] <= o) lo = mid + 1;
        else hi = mid;
    }
    tile_run[t] = lo - 1;
}

// ===========================================================================
// Host launchers
// ===========================================================================
size_t scan_ctl_bytes() { return align_up(sizeof(ScanCtl<512, 8>), 128); }   // >= every (NT, ITEMS) variant
size_t join_run_cache_bytes() { return align_up((size_t)(kThreads * kJoinItems + 1) * 20, 128); }
int scan_tile() { return kThreads * kScanItems; }
int join_expand_tile() { return kThreads * kJoinItems; }

size_t join_runs_smem(int key_type)
{
    const size_t w = type_width(key_type);
    return align_up((kRunItems * kWarps + 1) * 8, 128) + 2 * (size_t)(kRunT + kRunExt) * w + 2 * (size_t)kRunT * 4 +
           16 + (size_t)kRunT * w;
}

template <typename F>
static int occ(F f, size_t smem, int threads = kThreads)
{
    int n = 0;
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, f, threads, smem) != cudaSuccess)
        return 0;
    return n;
}

int chain_occupancy(int which, int nt, int items, size_t smem)
{
    switch (which) {
    case 0:
        if (nt == 512) return items == 8 ? occ(k_scan_chain<512, 8, false, false>, smem, 512 + kAuxThreads)
                                         : occ(k_scan_chain<512, 4, false, false>, smem, 512 + kAuxThreads);
        switch (items) {
        case 4: return occ(k_scan_chain<256, 4, false, false>, smem, 256 + kAuxThreads);
        case 5: return occ(k_scan_chain<256, 5, false, false>, smem, 256 + kAuxThreads);
        case 6: return occ(k_scan_chain<256, 6, false, false>, smem, 256 + kAuxThreads);
        default: return occ(k_scan_chain<256, 8, false, false>, smem, 256 + kAuxThreads);
        }
    case 4:   // input-dependence branches
        return items == 4 ? occ(k_scan_chain<256, 4, false, false, true>, smem, 256 + kAuxThreads)
                          : occ(k_scan_chain<256, 8, false, false, true>, smem, 256 + kAuxThreads);
    case 1:
        if (nt == 128) return occ(k_scan_chain<128, 16, true, false>, smem, 128 + 32);
        if (nt == 384) return occ(k_scan_chain<384, 5, true, false>, smem, 384 + 32);
        if (nt == 448) return occ(k_scan_chain<448, 4, true, false>, smem, 448 + 32);
        if (nt == 480) return occ(k_scan_chain<480, 4, true, false>, smem, 480 + 32);
        if (nt == kNarrowNT) return occ(k_scan_chain<kNarrowNT, kNarrowItems, true, false>, smem, kNarrowNT + 32);
        return items == 4 ? occ(k_scan_chain<256, 4, true, false>, smem, 256 + 32)
                          : occ(k_scan_chain<256, 8, true, false>, smem, 256 + 32);
    case 2: return occ(k_scan_chain<kThreads, kJoinItems, false, true>, smem, kThreads + kAuxThreads);
    default: return occ(k_join_runs<uint64_t, true>, smem);
    }
}

template <int NT, int ITEMS, bool AGG, bool MULTI = false>
static cudaError_t sc(const ChainProg &P, const TileLaunch &L, size_t smem, int grid, cudaStream_t s)
{
    JoinExpand X{};
    cudaFuncSetAttribute(k_scan_chain<NT, ITEMS, AGG, false, MULTI>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
    k_scan_chain<NT, ITEMS, AGG, false, MULTI><<<grid, NT + aux_threads(AGG), smem, s>>>(P, L, X);
    return cudaGetLastError();
}

cudaError_t join_chain_launch(const ChainProg &P, const TileLaunch &L, const JoinExpand &X, size_t smem, int grid,
                              cudaStream_t s)
{
    cudaFuncSetAttribute(k_scan_chain<kThreads, kJoinItems, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
    k_scan_chain<kThreads, kJoinItems, false, true><<<grid, kThreads + kAuxThreads, smem, s>>>(P, L, X);
    return cudaGetLastError();
}

cudaError_t scan_chain_launch(const ChainProg &P, const TileLaunch &L, bool agg, int nt, int items, size_t smem,
                              int grid, cudaStream_t s)
{
    if (!agg && P.nbranch > 1)
        return items == 4 ? sc<256, 4, false, true>(P, L, smem, grid, s) : sc<256, 8, false, true>(P, L, smem, grid, s);
    if (agg) {
        if (nt == 128)
            return sc<128, 16, true>(P, L, smem, grid, s);
        if (nt == 384)
            return sc<384, 5, true>(P, L, smem, grid, s);
        if (nt == 448)
            return sc<448, 4, true>(P, L, smem, grid, s);
        if (nt == 480)
            return sc<480, 4, true>(P, L, smem, grid, s);
        if (nt == kNarrowNT)
            return sc<kNarrowNT, kNarrowItems, true>(P, L, smem, grid, s);
        return items == 4 ? sc<256, 4, true>(P, L, smem, grid, s) : sc<256, 8, true>(P, L, smem, grid, s);
    }
    if (nt == 512)
        return items == 8 ? sc<512, 8, false>(P, L, smem, grid, s) : sc<512, 4, false>(P, L, smem, grid, s);
    switch (items) {
    case 4: return sc<256, 4, false>(P, L, smem, grid, s);
    case 5: return sc<256, 5, false>(P, L, smem, grid, s);
    case 6: return sc<256, 6, false>(P, L, smem, grid, s);
    default: return sc<256, 8, false>(P, L, smem, grid, s);
    }
}

cudaError_t agg_finalize_launch(const AggFinal &F, cudaStream_t s)
{
    k_agg_finalize<<<1, kThreads, 0, s>>>(F);
    return cudaGetLastError();
}

template <typename K>
static cudaError_t jr(const JoinRunsLaunch &J, size_t smem, int grid, cudaStream_t s)
{
    k_merge_splits<K><<<(unsigned)((J.nparts + 1 + 255) / 256), 256, 0, s>>>(J);
    cudaFuncSetAttribute(k_join_runs<K, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_join_runs<K, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (J.nparts > 0) {
        k_join_runs<K, false><<<grid, kThreads, smem, s>>>(J);
        k_scan_parts<<<1, 1024, 0, s>>>(J);
        k_join_runs<K, true><<<grid, kThreads, smem, s>>>(J);
    } else {
        k_scan_parts<<<1, 1024, 0, s>>>(J);
    }
    return cudaGetLastError();
}

cudaError_t join_runs_launch(const JoinRunsLaunch &J, int key_type, size_t smem, int grid, cudaStream_t s)
{
    switch (key_type) {
    case T_I32: return jr<int32_t>(J, smem, grid, s);
    case T_U32: return jr<uint32_t>(J, smem, grid, s);
    case T_I64: return jr<int64_t>(J, smem, grid, s);
    case T_U64: return jr<uint64_t>(J, smem, grid, s);
    default: return jr<uint8_t>(J, smem, grid, s);
    }
}

cudaError_t tile_runs_launch(const uint64_t *off, int64_t nruns, int64_t ntiles, int64_t T, int64_t *tile_run,
                             cudaStream_t s)
{
    if (ntiles > 0)
        k_tile_runs<<<(unsigned)((ntiles + 255) / 256), 256, 0, s>>>(off, nruns, ntiles, T, tile_run);
    return cudaGetLastError();
}


}  // namespace rw
