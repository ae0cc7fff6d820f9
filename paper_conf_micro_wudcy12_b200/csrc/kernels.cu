// kernels.cu — the sm_100a kernels of the fused relational-algebra hot path.
//
//   k_scan_chain<ITEMS, AGG>  fused SELECT / PROJECT / arithmetic chain over one
//                             input relation, terminal =
//                             compacted store or group-by aggregate (a9).
//   k_agg_finalize            128-bit accumulators -> output relation (groups with
//                             count > 0, ascending code).
//   (the compacting scan chains run on scan_emit.cu, the JOIN path on join2.cu;
//    this kernel carries the aggregate terminal and, opts.reserved[6] == 3, the
//    earlier L2-ring scan for comparison)
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

template <int NT, int ITEMS, bool AGG, bool MULTI = false>
__global__ void __launch_bounds__(NT + aux_threads(AGG), AGG ? 1 : 2) k_scan_chain(const __grid_constant__ ChainProg P,
                                                                     const __grid_constant__ TileLaunch L)
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
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t n = L.n_ptr ? *L.n_ptr : L.n;
    const int64_t ntiles = (n + T - 1) / T;
    const bool emit = !AGG && !(L.dbg & 2) && !L.direct;
    // input-dependence branches: only the MULTI instance carries the branch loop, so
    // the single-chain instances compile with NB == 1
    const int NB = (AGG || !MULTI) ? 1 : P.nbranch;

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
                if (t < ntiles && L.use_tma && (t + 1) * (int64_t)T <= n) {
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
            if (!(L.use_tma && rows == T)) {
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
            if constexpr (AGG && NT == kNarrowNT) {
                if (P.q1fused) {
                    // Q1 program shape: SELECT, arithmetic and aggregate fused per row
                    agg_tile_q1<NT, ITEMS>(P, st, mask0, racc, cta_acc, since_flush, L.err);
                    release_stage();
                    continue;
                }
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
// Host launchers
// ===========================================================================
size_t scan_ctl_bytes() { return align_up(sizeof(ScanCtl<512, 8>), 128); }   // >= every (NT, ITEMS) variant
int scan_tile() { return kThreads * kScanItems; }

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
        if (nt == 512) return items == 8 ? occ(k_scan_chain<512, 8, false>, smem, 512 + kAuxThreads)
                                         : occ(k_scan_chain<512, 4, false>, smem, 512 + kAuxThreads);
        switch (items) {
        case 4: return occ(k_scan_chain<256, 4, false>, smem, 256 + kAuxThreads);
        case 5: return occ(k_scan_chain<256, 5, false>, smem, 256 + kAuxThreads);
        case 6: return occ(k_scan_chain<256, 6, false>, smem, 256 + kAuxThreads);
        default: return occ(k_scan_chain<256, 8, false>, smem, 256 + kAuxThreads);
        }
    case 4:   // input-dependence branches
        return items == 4 ? occ(k_scan_chain<256, 4, false, true>, smem, 256 + kAuxThreads)
                          : occ(k_scan_chain<256, 8, false, true>, smem, 256 + kAuxThreads);
    case 1:
        if (nt == 128) return occ(k_scan_chain<128, 16, true>, smem, 128 + 32);
        if (nt == 384) return occ(k_scan_chain<384, 5, true>, smem, 384 + 32);
        if (nt == 448) return occ(k_scan_chain<448, 4, true>, smem, 448 + 32);
        if (nt == 480) return occ(k_scan_chain<480, 4, true>, smem, 480 + 32);
        if (nt == kNarrowNT) return occ(k_scan_chain<kNarrowNT, kNarrowItems, true>, smem, kNarrowNT + 32);
        return items == 4 ? occ(k_scan_chain<256, 4, true>, smem, 256 + 32)
                          : occ(k_scan_chain<256, 8, true>, smem, 256 + 32);
    default: return 0;
    }
}

template <int NT, int ITEMS, bool AGG, bool MULTI = false>
static cudaError_t sc(const ChainProg &P, const TileLaunch &L, size_t smem, int grid, cudaStream_t s)
{
    cudaFuncSetAttribute(k_scan_chain<NT, ITEMS, AGG, MULTI>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
    k_scan_chain<NT, ITEMS, AGG, MULTI><<<grid, NT + aux_threads(AGG), smem, s>>>(P, L);
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


}  // namespace rw
