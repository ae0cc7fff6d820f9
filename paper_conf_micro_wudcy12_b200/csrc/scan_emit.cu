// scan_emit.cu — the fused SELECT / PROJECT / arithmetic chain with a compacted
// output (patterns (a), (e) and, with branches, (d)).
//
// One persistent CTA per SM (or two), warp-specialised:
//   producer warp  claims tiles in order (one global atomic per tile, so the decoupled
//                  look-back always has forward progress) and stages every live column
//                  of the tile into shared memory with one TMA bulk copy per column
//                  (cp.async.bulk -> full[s]), S stages deep;
//   compute warps  run the fused program on the staged tile over 4-row vectors
//                  (chain4.cuh: one LDS.128 per 4 rows of a 4-byte column), count the
//                  survivors per warp with one packed shuffle scan, meet once per tile
//                  at a named barrier for the block prefix, publish the tile aggregate,
//                  and compact the survivors (tile order) into a byte ring in shared
//                  memory; the input stage is released at once, so the TMA pipeline
//                  never waits for a tile's global offset;
//   writer warps   (kWriters, round-robin over the compacted blocks) resolve each
//                  block's global offset by the decoupled look-back (chain.cuh) — the
//                  paper's separate gather stage — copy it to HBM with coalesced
//                  stores and release its ring bytes in order.
// Every wait is a suspending mbarrier try_wait (no polling loops in the aux warps);
// the only CTA-wide synchronisation per tile is the one compute barrier.
#include "chain4.cuh"
#include "kernels.h"

namespace rw {

constexpr int kEmitMaxStages = 8;
constexpr int kEmitMaxCnt = 64;           // G * NW counters per branch (G <= 4 groups of 4 rows, NW warps)
constexpr uint32_t kComputeBarEmit = 1;   // named barrier of the compute warps
constexpr int kWriters = 4;               // look-back + copy-out warps
constexpr int kEmitAux = 32 * (1 + kWriters);
constexpr int kEmitSlots = 16;            // compacted blocks in flight per CTA

struct EmitBlk {
    uint64_t aggr, oempty;                // block written (NW arrivals) / block copied out and released
    int64_t tile;
    uint32_t total, roff, used, br;
    uint32_t where;                       // 0: shared-memory ring, 1: L2 ring
};

struct EmitCtl {
    uint64_t full[kEmitMaxStages], empty[kEmitMaxStages];
    int64_t tile[kEmitMaxStages];
    EmitBlk blk[kEmitSlots];
    uint32_t cnt[4][kMaxBranch][kEmitMaxCnt];   // [team * 2 + parity of the team's tile]
    volatile uint32_t tail[2];                  // ring bytes released by the writers (monotone, wraps): smem, L2
    // two-team kernels: ring reservations are made in block order through this state
    // (slot i & 3 holds the (head, pos) of both rings before block i)
    volatile uint32_t rsv_seq;
    volatile uint32_t rsv[4][4];
};

static __host__ __device__ inline size_t al128e(size_t x) { return (x + 127) / 128 * 128; }
__device__ __forceinline__ uint32_t al16e(uint32_t x) { return (x + 15u) & ~15u; }

size_t emit_ctl_bytes() { return al128e(sizeof(EmitCtl)); }

// copy `total` elements of one compacted column (16-byte aligned in the ring) to
// dst[base ..): 16-byte shared loads, element-wide coalesced global stores (the
// destination offset is arbitrary); rows at or beyond `cap` are dropped
template <typename T, bool GR = false>
__device__ __forceinline__ void emit_copy(T *dst, const T *src, int64_t base, uint32_t total, int64_t cap, int lane)
{
    const int64_t lim = cap - base;
    const uint32_t m = (int64_t)total < lim ? total : (lim > 0 ? (uint32_t)lim : 0u);
    T *d = dst + base;
    uint32_t j0 = 0;
    if (sizeof(T) >= 4) {
        // 16-byte loads, U of them in flight per lane (an L2 ring is ~1 us away)
        constexpr int V = 16 / sizeof(T);
        constexpr int U = GR ? 8 : 2;
        const uint4 *s4 = (const uint4 *)src;
        const uint32_t nv = m / V;
        uint32_t j = lane;
        for (; j + (U - 1) * 32 < nv; j += U * 32) {
            uint4 v[U];
#pragma unroll
            for (int u = 0; u < U; u++)
                v[u] = GR ? __ldcg(s4 + j + u * 32) : s4[j + u * 32];
#pragma unroll
            for (int u = 0; u < U; u++) {
                const T *e = (const T *)&v[u];
#pragma unroll
                for (int x = 0; x < V; x++)
                    d[(size_t)(j + u * 32) * V + x] = e[x];
            }
        }
        for (; j < nv; j += 32) {
            const uint4 v = GR ? __ldcg(s4 + j) : s4[j];
            const T *e = (const T *)&v;
#pragma unroll
            for (int x = 0; x < V; x++)
                d[(size_t)j * V + x] = e[x];
        }
        j0 = nv * V;
    }
    for (uint32_t j = j0 + lane; j < m; j += 32)
        d[j] = GR ? __ldcg(src + j) : src[j];
}

// The survivors (positions sp) of columns [c0, c1) of the staged tile into a compacted
// block at byte `pos` of a circular ring of R bytes (shared or global: inlined per call
// site, so each gets plain STS or STG); a column segment that wraps takes the slow path.
template <int NT, int G, bool GR = false>
__device__ __forceinline__ void compact_block(const ChainProg &P, int c0, int c1, const char *st, const char *scratch,
                                              uint32_t m, const uint32_t (&sp)[G][4], uint32_t total, char *ring,
                                              uint32_t R, uint32_t pos)
{
    const uint64_t pol = GR ? policy_evict_last() : 0ull;
    uint32_t coff = 0;
    for (int c = c0; c < c1; c++) {
        const int w = P.out_w[c];
        const char *src = loc_ptr(P.out_loc[c], st, scratch);
        const uint32_t so = pos + coff >= R ? pos + coff - R : pos + coff;   // pos, coff < R
        coff += al16e(total * w);
        if (so + total * (uint32_t)w > R) {
            wrap_scatter<NT, G>(ring, R, so, w, src, m, sp);
            continue;
        }
        char *d = ring + so;
        if (w == 4) {
#pragma unroll
            for (int g = 0; g < G; g++) {
                const uint32_t m4 = (m >> (4 * g)) & 15u;
                if (!m4)
                    continue;
                const V4<uint32_t> x = ld4<uint32_t>(src, row4<NT>(g));
#pragma unroll
                for (int q = 0; q < 4; q++)
                    if ((m4 >> q) & 1u) { if (GR) st_l2keep((uint32_t *)d + sp[g][q], x.v[q], pol); else ((uint32_t *)d)[sp[g][q]] = x.v[q]; }
            }
        } else if (w == 8) {
#pragma unroll
            for (int g = 0; g < G; g++) {
                const uint32_t m4 = (m >> (4 * g)) & 15u;
                if (!m4)
                    continue;
                const V4<uint64_t> x = ld4<uint64_t>(src, row4<NT>(g));
#pragma unroll
                for (int q = 0; q < 4; q++)
                    if ((m4 >> q) & 1u) { if (GR) st_l2keep((uint64_t *)d + sp[g][q], x.v[q], pol); else ((uint64_t *)d)[sp[g][q]] = x.v[q]; }
            }
        } else {
#pragma unroll
            for (int g = 0; g < G; g++) {
                const uint32_t m4 = (m >> (4 * g)) & 15u;
                if (!m4)
                    continue;
                const V4<uint8_t> x = ld4<uint8_t>(src, row4<NT>(g));
#pragma unroll
                for (int q = 0; q < 4; q++)
                    if ((m4 >> q) & 1u) { if (GR) st_l2keep((uint8_t *)d + sp[g][q], x.v[q], pol); else ((uint8_t *)d)[sp[g][q]] = x.v[q]; }
            }
        }
    }
}

// Compacted tiles wait in one of two circular rings: small blocks in shared memory, blocks
// larger than a quarter of it (high-selectivity chains) in a per-CTA slice of an
// L2-resident global buffer, so that enough tiles stay in flight for any selectivity.
// The choice depends only on the block size, so every compute warp makes the same one.
//
// TEAMS = 2: the compute warps form two teams of NT threads that take alternate tiles
// (team = stage use mod 2), each with its own named barrier and count buffers, so one
// team's barrier, prefix and compaction overlap the other's evaluation; the compacted
// blocks still reserve their ring bytes in tile order (ctl->rsv_seq).
template <int NT, int ITEMS, bool MULTI, int TEAMS = 1>
__global__ void __launch_bounds__(NT * TEAMS + kEmitAux, 1) k_scan_emit(const __grid_constant__ ChainProg P,
                                                                       const __grid_constant__ TileLaunch L)
{
    constexpr int G = ITEMS / 4;
    constexpr int T = NT * ITEMS;
    constexpr int NW = NT / 32;                 // compute warps per team
    constexpr int NWC = NW * TEAMS;             // compute warps
    static_assert(TEAMS == 1 || !MULTI, "two-team kernel: single chain only");
    static_assert(ITEMS % 4 == 0 && G <= 4 && G * NW <= kEmitMaxCnt, "emit tile geometry");
    constexpr int NBR = MULTI ? kMaxBranch : 1;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    EmitCtl *ctl = (EmitCtl *)smem_raw;
    const int S = L.stages;
    const uint32_t SB = P.stage_bytes;
    char *stages = (char *)smem_raw + al128e(sizeof(EmitCtl));
    char *scratch = stages + (size_t)S * SB;              // computed columns of the tile being evaluated
    const uint32_t Rs = L.out_bytes;                      // shared ring bytes (multiple of 128, may be 0)
    const uint32_t Rg = L.gring ? L.gring_bytes : 0u;     // L2 ring bytes per CTA (0: none)
    char *ring_s = scratch + P.scratch_bytes;
    char *ring_g = L.gring ? L.gring + (size_t)blockIdx.x * Rg : nullptr;
    const int NB = MULTI ? P.nbranch : 1;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int64_t n = L.n_ptr ? *L.n_ptr : L.n;
    const int64_t ntiles = (n + T - 1) / T;
    const uint32_t full_mask = ITEMS == 32 ? 0xffffffffu : (1u << ITEMS) - 1u;
    const bool emit = !L.direct && !(L.dbg & 2);

    if (tid == 0) {
        for (int s = 0; s < S; s++) {
            mbar_init(&ctl->full[s], 1);
            mbar_init(&ctl->empty[s], NW);             // one arrival per compute warp
        }
        for (int j = 0; j < kEmitSlots; j++) {
            mbar_init(&ctl->blk[j].aggr, NW);          // one arrival per compute warp
            mbar_init(&ctl->blk[j].oempty, 1);
        }
        ctl->tail[0] = 0;
        ctl->tail[1] = 0;
        ctl->rsv_seq = 0;
        for (int q = 0; q < 4; q++)
            ctl->rsv[0][q] = 0;
        fence_mbar_init();
    }
    __syncthreads();

    if (warp == NWC) {
        // ---------------- producer warp ----------------
        if (lane == 0) {
            uint32_t tx_bytes = 0;
            for (int i = 0; i < P.nin; i++)
                tx_bytes += (uint32_t)T * type_width(P.slot[i].type);
            const uint64_t policy = policy_evict_first();
            // the next tile is claimed one stage ahead, so the atomic's round trip overlaps
            // the wait for a free stage (a claimed tile depends only on tiles claimed
            // before it, so holding the claim cannot stall any look-back cycle)
            int64_t tn = (int64_t)atomicAdd(&L.ctrs[0], 1u);
            int s = 0;
            uint32_t eph = 1;                               // parity of the stage's previous use
            int sentinels = 0;                              // one per team (tile = ntiles + team-order)
            for (uint32_t i = 0;; ++i) {
                const int64_t t = tn >= ntiles ? ntiles + sentinels : tn;
                if (tn < ntiles)
                    tn = (int64_t)atomicAdd(&L.ctrs[0], 1u);
                if (i >= (uint32_t)S)
                    mbar_wait(&ctl->empty[s], eph);
                ctl->tile[s] = t;
                if (t < ntiles && L.use_tma && (t + 1) * (int64_t)T <= n) {
                    char *st = stages + (size_t)s * SB;
                    fence_proxy_async_smem();
                    mbar_arrive_expect_tx(&ctl->full[s], tx_bytes);
                    for (int c = 0; c < P.nin; c++) {
                        const int w = type_width(P.slot[c].type);
                        bulk_g2s(st + P.slot[c].off, (const char *)P.in_ptr[c] + (size_t)t * T * w, (uint32_t)T * w,
                                 &ctl->full[s], policy);
                    }
                } else {
                    mbar_arrive(&ctl->full[s]);
                }
                if (t >= ntiles && ++sentinels == TEAMS)
                    break;
                if (++s == S) {
                    s = 0;
                    eph ^= 1u;
                }
            }
        }
    } else if (warp > NWC) {
        // ---------------- writer warps: look-back + copy-out, block i = wi mod kWriters ----------------
        const int wi = warp - NWC - 1;
        if (emit) {
            for (uint32_t i = wi;; i += kWriters) {
                const int j = (int)(i % kEmitSlots);
                mbar_wait(&ctl->blk[j].aggr, (i / kEmitSlots) & 1u);
                const int64_t t = ctl->blk[j].tile;
                if (t >= ntiles)
                    break;
                const uint32_t total = ctl->blk[j].total;
                const int b = (int)ctl->blk[j].br;
                const int64_t excl = (L.dbg & 1) ? t * T
                                                 : (int64_t)lookback_warp(L.status + b * L.status_stride, t, total, L.epoch,
                                                                          /*aggregate_published=*/true,
                                                                          (L.dbg & 128) ? 0u : (L.dbg & 64) ? 256u : 1024u);
                if (lane == 0 && t == ntiles - 1)
                    *(b ? L.br_n_dev[b] : L.n_dev) = excl + (int64_t)total;
                const uint32_t roff = ctl->blk[j].roff;
                const int64_t cap = b ? P.br_cap[b] : P.out_capacity;
                const int where = (int)ctl->blk[j].where;
                const uint32_t R = where ? Rg : Rs;
                const char *ring = where ? ring_g : ring_s;
                uint32_t coff = 0;
                for (int c = b ? P.br_out_end[b - 1] : 0; c < (MULTI ? (int)P.br_out_end[b] : P.nout); c++) {
                    const int w = P.out_w[c];
                    // the ring is circular: a column's segment may wrap at R (16-byte
                    // aligned, so no vector straddles the end) -> copied in two pieces
                    const uint32_t so = roff + coff >= R ? roff + coff - R : roff + coff;   // roff, coff < R
                    coff += al16e(total * w);
                    const uint32_t n1 = min(total, (R - so) / (uint32_t)w);
                    for (int piece = 0; piece < 2; piece++) {
                        const char *src = piece ? ring : ring + so;
                        const int64_t at = piece ? excl + n1 : excl;
                        const uint32_t cnt = piece ? total - n1 : n1;
                        if (cnt == 0) continue;
                        if (where) {
                            if (w == 4) emit_copy<uint32_t, true>((uint32_t *)P.out_ptr[c], (const uint32_t *)src, at, cnt, cap, lane);
                            else if (w == 8) emit_copy<uint64_t, true>((uint64_t *)P.out_ptr[c], (const uint64_t *)src, at, cnt, cap, lane);
                            else emit_copy<uint8_t, true>((uint8_t *)P.out_ptr[c], (const uint8_t *)src, at, cnt, cap, lane);
                        } else {
                            if (w == 4) emit_copy<uint32_t>((uint32_t *)P.out_ptr[c], (const uint32_t *)src, at, cnt, cap, lane);
                            else if (w == 8) emit_copy<uint64_t>((uint64_t *)P.out_ptr[c], (const uint64_t *)src, at, cnt, cap, lane);
                            else emit_copy<uint8_t>((uint8_t *)P.out_ptr[c], (const uint8_t *)src, at, cnt, cap, lane);
                        }
                    }
                }
                __syncwarp();
                if (where) {
                    // the block is copied out: drop its fully covered L2 lines, so the ring
                    // never costs a DRAM write-back
                    const uint32_t used_b = ctl->blk[j].used;
                    for (uint32_t o = ((roff + 127u) & ~127u) + (uint32_t)lane * 128u; o + 128u <= roff + used_b; o += 32u * 128u)
                        if (o + 128u <= R) discard_l2_line(ring_g + o);
                    __syncwarp();
                }
                if (lane == 0) {
                    if (i > 0)   // ring bytes are released in block order
                        mbar_wait(&ctl->blk[(i - 1) % kEmitSlots].oempty, ((i - 1) / kEmitSlots) & 1u);
                    if (where)
                        __threadfence();   // the discards land before the bytes are rewritten
                    else
                        __threadfence_block();
                    ctl->tail[where] = ctl->tail[where] + ctl->blk[j].used;
                    mbar_arrive(&ctl->blk[j].oempty);
                }
                __syncwarp();
            }
        }
    } else {
        // ---------------- compute warps ----------------
        const int team = TEAMS > 1 ? warp / NW : 0;
        const int ltid = tid - team * NT, lwarp = warp - team * NW;   // within the team
        uint32_t head_s = 0, hpos_s = 0, head_g = 0, hpos_g = 0;   // ring reservations, replicated in every warp
        for (uint32_t i = team;; i += TEAMS) {
            const int s = (int)(i % (uint32_t)S);
            const uint32_t fph = (i / (uint32_t)S) & 1u;
            uint32_t ublk = i * (uint32_t)NB;                // compacted blocks before this tile's (tile order)
            mbar_wait(&ctl->full[s], fph);
            const int64_t t = ctl->tile[s];
            if (t >= ntiles) {
                // the first sentinel's team sends one sentinel block per writer warp
                // (consecutive slots after every real block)
                if (emit && ltid == 0 && t == ntiles) {
                    for (uint32_t u = ublk; u < ublk + kWriters; ++u) {
                        const int ju = (int)(u % kEmitSlots);
                        if (u >= kEmitSlots)
                            mbar_wait(&ctl->blk[ju].oempty, ((u / kEmitSlots) - 1) & 1u);
                        ctl->blk[ju].tile = ntiles;
                        mbar_arrive_cnt(&ctl->blk[ju].aggr, NW);
                    }
                }
                break;
            }
            char *st = stages + (size_t)s * SB;
            const int64_t row0 = t * T;
            const int rows = (int)min((int64_t)T, n - row0);
            if (!(L.use_tma && rows == T)) {
                // ragged last tile or unaligned bases: each thread loads its own rows
                for (int c = 0; c < P.nin; c++) {
                    const int w = type_width(P.slot[c].type);
                    char *dst = st + P.slot[c].off;
                    const char *src = (const char *)P.in_ptr[c] + (size_t)row0 * w;
#pragma unroll
                    for (int g = 0; g < G; g++)
#pragma unroll
                        for (int q = 0; q < 4; q++) {
                            const int r = row4<NT>(g) + q;
                            if (r < rows) {
                                if (w == 4) ((uint32_t *)dst)[r] = ((const uint32_t *)src)[r];
                                else if (w == 8) ((uint64_t *)dst)[r] = ((const uint64_t *)src)[r];
                                else dst[r] = src[r];
                            }
                        }
                }
            }
            uint32_t mask0 = full_mask;
            if (rows < T) {
                mask0 = 0;
#pragma unroll
                for (int g = 0; g < G; g++)
#pragma unroll
                    for (int q = 0; q < 4; q++)
                        if (row4<NT>(g) + q < rows)
                            mask0 |= 1u << (g * 4 + q);
            }
            if (!emit) {
                if (L.direct && !(L.dbg & 2)) {
                    // no SELECT in the group: every row is stored at its own row offset
                    run_ops4<NT, G>(P, 0, P.nops, st, scratch, mask0);
                    const int64_t cap = P.out_capacity;
                    for (int c = 0; c < P.nout; c++) {
                        const int w = P.out_w[c];
                        const char *src = loc_ptr(P.out_loc[c], st, scratch);
#pragma unroll
                        for (int g = 0; g < G; g++) {
                            const int r0 = row4<NT>(g);
#pragma unroll
                            for (int q = 0; q < 4; q++) {
                                const int64_t gr = row0 + r0 + q;
                                if (r0 + q < rows && gr < cap) {
                                    if (w == 4) ((uint32_t *)P.out_ptr[c])[gr] = ((const uint32_t *)src)[r0 + q];
                                    else if (w == 8) ((uint64_t *)P.out_ptr[c])[gr] = ((const uint64_t *)src)[r0 + q];
                                    else ((uint8_t *)P.out_ptr[c])[gr] = ((const uint8_t *)src)[r0 + q];
                                }
                            }
                        }
                    }
                }
                __syncwarp();
                if (lane == 0)
                    mbar_arrive(&ctl->empty[s]);
                continue;
            }
            // evaluate every branch: survivor masks and per-warp counts of each 4-row group
            // (a second branch recomputes into the same scratch, so branches are evaluated
            // and compacted one after the other; branch b's counts are published first)
            const int par = TEAMS > 1 ? team * 2 + (int)((i / TEAMS) & 1u) : (int)(i & 1u);
            for (int b = 0; b < NB; b++) {
                const uint32_t m = run_ops4<NT, G>(P, b ? (int)P.br_op_end[b - 1] : 0, MULTI ? (int)P.br_op_end[b] : P.nops,
                                                   st, scratch, mask0);
                // survivors per 4-row group, packed 8 bits per group (a warp's group count <= 128)
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
                        ctl->cnt[par][b][g * NW + lwarp] = (inc >> (8 * g)) & 255u;
                const uint32_t ex = inc - pk;
                bar_sync(kComputeBarEmit + team, NT);
                // block prefix of (group, warp) in tile order and the tile total (G * NW
                // counters: one per lane, or two when there are more than 32)
                constexpr int GN = G * NW;
                const uint32_t v = lane < GN ? ctl->cnt[par][b][lane] : 0u;
                uint32_t bin = v;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, bin, o);
                    if (lane >= o)
                        bin += y;
                }
                uint32_t total = __shfl_sync(0xffffffffu, bin, 31);
                uint32_t v2 = 0, bin2 = 0;
                const uint32_t total0 = total;
                if constexpr (GN > 32) {
                    v2 = lane + 32 < GN ? ctl->cnt[par][b][lane + 32] : 0u;
                    bin2 = v2;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const uint32_t y = __shfl_up_sync(0xffffffffu, bin2, o);
                        if (lane >= o)
                            bin2 += y;
                    }
                    total = total0 + __shfl_sync(0xffffffffu, bin2, 31);
                }
                uint32_t pre[G];
#pragma unroll
                for (int g = 0; g < G; g++) {
                    const int idx = g * NW + lwarp;
                    uint32_t e;
                    if constexpr (GN > 32) {
                        const uint32_t e0 = __shfl_sync(0xffffffffu, bin - v, idx & 31);
                        const uint32_t e1 = __shfl_sync(0xffffffffu, bin2 - v2, idx & 31) + total0;
                        e = idx < 32 ? e0 : e1;
                    } else {
                        e = __shfl_sync(0xffffffffu, bin - v, idx);
                    }
                    pre[g] = e + ((ex >> (8 * g)) & 255u);
                }
                if (lwarp == 0 && lane == 0 && t > 0 && !(L.dbg & 1))
                    // publish the tile aggregate before anything can block this CTA
                    st_relaxed_u64(&L.status[b * L.status_stride + t], ((uint64_t)L.epoch << 48) | (1ull << 46) | total);
                // ring bytes of the compacted block (blocks never wrap); every warp computes
                // the same reservation from the same (head, hpos, total)
                const int c0 = b ? P.br_out_end[b - 1] : 0, c1 = MULTI ? (int)P.br_out_end[b] : P.nout;
                const uint32_t need = P.br_nw[b][0] * al16e(total) + P.br_nw[b][1] * al16e(total * 4u) +
                                      P.br_nw[b][2] * al16e(total * 8u);
                // circular rings: the block goes to the shared ring unless it is larger than a
                // quarter of it (then to the L2 ring); wait until its bytes are free
                const int where = Rg != 0u && (Rs == 0u || need > Rs / 4u) ? 1 : 0;
                const uint32_t R = where ? Rg : Rs;
                const uint32_t used = need;
                if constexpr (TEAMS > 1) {
                    // the other team reserves the blocks in between: take the ring state
                    // left by block ublk - 1 (slot ublk & 3 is not rewritten before every
                    // warp of this team has passed its next barrier)
                    if (lane == 0)
                        while (ctl->rsv_seq < ublk)
                            __nanosleep(20);
                    __syncwarp();
                    const uint32_t sl = ublk & 3u;
                    head_s = ctl->rsv[sl][0];
                    hpos_s = ctl->rsv[sl][1];
                    head_g = ctl->rsv[sl][2];
                    hpos_g = ctl->rsv[sl][3];
                }
                const uint32_t pos = where ? hpos_g : hpos_s;
                const uint32_t hd = where ? head_g : head_s;
                const int j = (int)(ublk % kEmitSlots);
                if (ublk >= kEmitSlots)
                    mbar_wait(&ctl->blk[j].oempty, ((ublk / kEmitSlots) - 1) & 1u);
                {
                    uint32_t backoff = 64;
                    while (hd + used - (where ? ctl->tail[1] : ctl->tail[0]) > R) {
                        __nanosleep(backoff);
                        backoff = backoff < 1024 ? backoff * 2 : 1024;
                    }
                }
                const uint32_t np = pos + need >= R ? pos + need - R : pos + need;
                if (where) { head_g = hd + used; hpos_g = np; }
                else { head_s = hd + used; hpos_s = np; }
                if constexpr (TEAMS > 1) {
                    if (lwarp == 0 && lane == 0) {
                        const uint32_t sl = (ublk + 1) & 3u;
                        ctl->rsv[sl][0] = head_s;
                        ctl->rsv[sl][1] = hpos_s;
                        ctl->rsv[sl][2] = head_g;
                        ctl->rsv[sl][3] = hpos_g;
                        __threadfence_block();
                        ctl->rsv_seq = ublk + 1;
                    }
                }
                // compact the survivors into the block, tile order: each surviving row's
                // position is computed once, then every column stores with it
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
                if (where)
                    compact_block<NT, G, true>(P, c0, c1, st, scratch, m, sp, total, ring_g, R, pos);
                else
                    compact_block<NT, G>(P, c0, c1, st, scratch, m, sp, total, ring_s, R, pos);
                __syncwarp();
                if (lane == 0) {
                    if (where)
                        __threadfence_block();
                    if (lwarp == 0) {
                        ctl->blk[j].tile = t;
                        ctl->blk[j].total = total;
                        ctl->blk[j].roff = pos;
                        ctl->blk[j].used = used;
                        ctl->blk[j].br = (uint32_t)b;
                        ctl->blk[j].where = (uint32_t)where;
                    }
                    if (b == NB - 1)
                        mbar_arrive(&ctl->empty[s]);      // this warp is done with the stage
                    mbar_arrive(&ctl->blk[j].aggr);       // and with the compacted block
                }
                ++ublk;
            }
        }
    }
    __syncthreads();
    if (blockIdx.x == 0 && tid == 0 && (ntiles == 0 || L.direct)) {
        *L.n_dev = L.direct ? n : 0;
        for (int b = 1; b < NB; b++)
            *L.br_n_dev[b] = 0;
    }
    cta_exit_reset(L.ctrs);
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
template <int NT, int ITEMS, bool MULTI, int TEAMS = 1>
static int emit_occ(size_t smem)
{
    auto f = k_scan_emit<NT, ITEMS, MULTI, TEAMS>;
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, f, NT * TEAMS + kEmitAux, smem) != cudaSuccess)
        return 0;
    return n;
}

int scan_emit_occupancy(int nt, int items, bool multi, size_t smem, int teams)
{
    if (teams == 2)
        return nt == 128 ? emit_occ<128, 16, false, 2>(smem) : emit_occ<256, 8, false, 2>(smem);
    if (multi)
        return items == 4 ? emit_occ<256, 4, true>(smem) : emit_occ<256, 8, true>(smem);
    if (nt == 512)
        return emit_occ<512, 8, false>(smem);
    if (nt == 384)
        return items == 16 ? emit_occ<384, 16, false>(smem) : emit_occ<384, 8, false>(smem);
    return items == 4 ? emit_occ<256, 4, false>(smem) : items == 16 ? emit_occ<256, 16, false>(smem)
                                                      : emit_occ<256, 8, false>(smem);
}

template <int NT, int ITEMS, bool MULTI, int TEAMS = 1>
static cudaError_t emit_go(const ChainProg &P, const TileLaunch &L, size_t smem, int grid, cudaStream_t s)
{
    cudaFuncSetAttribute(k_scan_emit<NT, ITEMS, MULTI, TEAMS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    k_scan_emit<NT, ITEMS, MULTI, TEAMS><<<grid, NT * TEAMS + kEmitAux, smem, s>>>(P, L);
    return cudaGetLastError();
}

cudaError_t scan_emit_launch(const ChainProg &P, const TileLaunch &L, int nt, int items, size_t smem, int grid,
                             cudaStream_t s, int teams)
{
    if (teams == 2 && P.nbranch == 1)
        return nt == 128 ? emit_go<128, 16, false, 2>(P, L, smem, grid, s) : emit_go<256, 8, false, 2>(P, L, smem, grid, s);
    if (P.nbranch > 1)
        return items == 4 ? emit_go<256, 4, true>(P, L, smem, grid, s) : emit_go<256, 8, true>(P, L, smem, grid, s);
    if (nt == 512)
        return emit_go<512, 8, false>(P, L, smem, grid, s);
    if (nt == 384)
        return items == 16 ? emit_go<384, 16, false>(P, L, smem, grid, s) : emit_go<384, 8, false>(P, L, smem, grid, s);
    return items == 4 ? emit_go<256, 4, false>(P, L, smem, grid, s)
                      : items == 16 ? emit_go<256, 16, false>(P, L, smem, grid, s) : emit_go<256, 8, false>(P, L, smem, grid, s);
}

}  // namespace rw
