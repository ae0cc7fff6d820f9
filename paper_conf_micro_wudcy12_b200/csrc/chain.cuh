// chain.cuh — device side of a fused group: the per-tile micro-op interpreter
// (SELECT atoms, PROJECT / arithmetic), warp-ballot compaction, block scan,
// decoupled look-back, compacted store, and the group-by aggregate terminal.
//
// Tile layout: T = NT * ITEMS rows; thread `tid` owns rows k*NT+tid
// (k < ITEMS), so every smem slot access and every global store of a warp is
// over 32 consecutive rows.  The per-row predicate result is one bit of the
// register `mask` (§5.1.1: filters AND-ed into `match`).
#pragma once
#include "internal.h"
#include "ptx.cuh"

namespace rw {

constexpr int kWarps = kThreads / 32;

// ---------------------------------------------------------------------------
// Decoupled look-back (single-pass prefix over tiles) — replaces the paper's
// separate gather stage (§3 "gathered into a global dense sorted array").
// Status word: [epoch:16][flag:2][value:46]; flag 1 = aggregate, 2 = inclusive.
// Called by all 32 lanes of one warp; returns the tile's exclusive prefix and
// publishes its inclusive prefix.
// ---------------------------------------------------------------------------
constexpr uint64_t kValMask = (1ull << 46) - 1;

__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
        v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__device__ inline uint64_t lookback_warp(uint64_t *status, int64_t tile, uint64_t agg, uint32_t epoch,
                                         bool aggregate_published = false, uint32_t max_backoff = 1024)
{
    const int lane = threadIdx.x & 31;
    const uint64_t tag = (uint64_t)epoch << 48;
    if (tile == 0) {
        if (lane == 0)
            st_relaxed_u64(&status[0], tag | (2ull << 46) | agg);
        return 0;
    }
    if (lane == 0 && !aggregate_published)
        st_relaxed_u64(&status[tile], tag | (1ull << 46) | agg);
    // Each round inspects 128 predecessors (4 status words per lane): with ~10^2
    // tiles completing per microsecond chip-wide, a 32-wide window would let the
    // band of aggregate-only tiles outgrow one round and the walk would never settle.
    constexpr int Q = 4;
    uint64_t excl = 0;
    int64_t j = tile - 1;
    while (true) {
        uint64_t w[Q];
        uint32_t pending = 0;
#pragma unroll
        for (int q = 0; q < Q; q++) {
            const int64_t idx = j - lane * Q - q;
            w[q] = idx >= 0 ? ld_relaxed_u64(&status[idx]) : ((uint64_t)epoch << 48) | (2ull << 46);
            if ((uint32_t)(w[q] >> 48) != epoch || ((w[q] >> 46) & 3u) == 0)
                pending |= 1u << q;
        }
        uint32_t backoff = 32;
        while (pending) {
            // back off: hundreds of look-back warps polling the same few status
            // lines would otherwise starve the stores that publish them
            if (max_backoff)
                __nanosleep(backoff);
            backoff = backoff < max_backoff ? backoff * 2 : max_backoff;
#pragma unroll
            for (int q = 0; q < Q; q++) {
                if ((pending >> q) & 1u) {
                    w[q] = ld_relaxed_u64(&status[j - lane * Q - q]);
                    if ((uint32_t)(w[q] >> 48) == epoch && ((w[q] >> 46) & 3u) != 0)
                        pending &= ~(1u << q);
                }
            }
        }
        int firstq = Q;                             // nearest inclusive prefix within this lane
#pragma unroll
        for (int q = Q - 1; q >= 0; q--)
            if (((w[q] >> 46) & 3u) == 2u)
                firstq = q;
        const uint32_t pmask = __ballot_sync(0xffffffffu, firstq < Q);
        uint64_t s = 0;
        if (pmask) {
            const int first = __ffs(pmask) - 1;     // nearest lane holding an inclusive prefix
            if (lane < first) {
#pragma unroll
                for (int q = 0; q < Q; q++) s += w[q] & kValMask;
            } else if (lane == first) {
#pragma unroll
                for (int q = 0; q < Q; q++)
                    if (q <= firstq) s += w[q] & kValMask;
            }
            excl += warp_sum_u64(s);
            break;
        }
#pragma unroll
        for (int q = 0; q < Q; q++) s += w[q] & kValMask;
        excl += warp_sum_u64(s);
        j -= 32 * Q;
    }
    if (lane == 0)
        st_relaxed_u64(&status[tile], tag | (2ull << 46) | (excl + agg));
    return excl;
}

// Persistent kernels claim work items in order with ctrs[0] (so a decoupled look-back
// always has forward progress, whatever number of CTAs is resident); the last CTA to
// leave resets both counters for the next launch.
__device__ inline void cta_exit_reset(uint32_t *ctrs)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        if (atomicAdd(&ctrs[1], 1u) == gridDim.x - 1) {
            ctrs[0] = 0;
            ctrs[1] = 0;
            __threadfence();
        }
    }
}

// ---------------------------------------------------------------------------
// Slot access.  Locations are resolved on the host (kLocScratch | byte offset),
// so the interpreter never walks a slot table on the device.
// ---------------------------------------------------------------------------
__device__ __forceinline__ const char *loc_ptr(uint32_t loc, const char *stage, const char *scratch)
{
    return ((loc & kLocScratch) ? scratch : stage) + (loc & ~kLocScratch);
}

__device__ __forceinline__ const char *slot_ptr(const ChainProg &P, int s, const char *stage, const char *scratch)
{
    return (P.slot[s].is_input ? stage : scratch) + P.slot[s].off;
}

// Value of a slot row sign/zero-extended to 64 bits (its mathematical value mod 2^64).
__device__ __forceinline__ uint64_t ld_ext(const char *base, int type, int row)
{
    switch (type) {
    case T_I32: return (uint64_t)(int64_t)((const int32_t *)base)[row];
    case T_U32: return ((const uint32_t *)base)[row];
    case T_U8: return ((const uint8_t *)base)[row];
    default: return ((const uint64_t *)base)[row];
    }
}

template <typename T>
__device__ __forceinline__ T ld_as(const char *base, int row)
{
    return ((const T *)base)[row];
}

template <typename T, int CMP>
__device__ __forceinline__ bool cmpv(T x, T y)
{
    if (CMP == C_LT) return x < y;
    if (CMP == C_LE) return x <= y;
    if (CMP == C_GT) return x > y;
    if (CMP == C_GE) return x >= y;
    if (CMP == C_EQ) return x == y;
    return x != y;
}

// SELECT atom over the tile: clears bits of rows failing `a CMP b` (reading A4).
template <int NT, int ITEMS, typename T, int CMP, bool BSLOT>
__device__ __forceinline__ uint32_t pred_loop(const char *a, const char *b, T k, uint32_t mask)
{
    const int tid = threadIdx.x;
    const T *pa = (const T *)a;
    const T *pb = (const T *)b;
    uint32_t keep = 0;
#pragma unroll
    for (int i = 0; i < ITEMS; i++) {
        const T x = pa[i * NT + tid];
        const T y = BSLOT ? pb[i * NT + tid] : k;
        keep |= (uint32_t)cmpv<T, CMP>(x, y) << i;
    }
    return mask & keep;
}

#define RW_PRED_CASES(TT, TCODE)                                                                        \
    case TCODE * 8 + C_LT: return pred_loop<NT, ITEMS, TT, C_LT, false>(a, b, (TT)k, mask);             \
    case TCODE * 8 + C_LE: return pred_loop<NT, ITEMS, TT, C_LE, false>(a, b, (TT)k, mask);             \
    case TCODE * 8 + C_GT: return pred_loop<NT, ITEMS, TT, C_GT, false>(a, b, (TT)k, mask);             \
    case TCODE * 8 + C_GE: return pred_loop<NT, ITEMS, TT, C_GE, false>(a, b, (TT)k, mask);             \
    case TCODE * 8 + C_EQ: return pred_loop<NT, ITEMS, TT, C_EQ, false>(a, b, (TT)k, mask);             \
    case TCODE * 8 + C_NE: return pred_loop<NT, ITEMS, TT, C_NE, false>(a, b, (TT)k, mask);             \
    case 64 + TCODE * 8 + C_LT: return pred_loop<NT, ITEMS, TT, C_LT, true>(a, b, (TT)0, mask);         \
    case 64 + TCODE * 8 + C_LE: return pred_loop<NT, ITEMS, TT, C_LE, true>(a, b, (TT)0, mask);         \
    case 64 + TCODE * 8 + C_GT: return pred_loop<NT, ITEMS, TT, C_GT, true>(a, b, (TT)0, mask);         \
    case 64 + TCODE * 8 + C_GE: return pred_loop<NT, ITEMS, TT, C_GE, true>(a, b, (TT)0, mask);         \
    case 64 + TCODE * 8 + C_EQ: return pred_loop<NT, ITEMS, TT, C_EQ, true>(a, b, (TT)0, mask);         \
    case 64 + TCODE * 8 + C_NE: return pred_loop<NT, ITEMS, TT, C_NE, true>(a, b, (TT)0, mask);

template <int NT, int ITEMS>
__device__ __noinline__ uint32_t run_pred(uint32_t code, int64_t k, const char *a, const char *b, uint32_t mask)
{
    switch (code) {
        RW_PRED_CASES(int32_t, T_I32)
        RW_PRED_CASES(uint32_t, T_U32)
        RW_PRED_CASES(int64_t, T_I64)
        RW_PRED_CASES(uint64_t, T_U64)
        RW_PRED_CASES(uint8_t, T_U8)
    }
    return mask;
}

// Arithmetic in type T with wrap-around (reading A8): done in the unsigned twin.
template <typename T, int OP>
__device__ __forceinline__ T ev(T a, T b)
{
    typedef typename std::make_unsigned<T>::type U;
    if (OP == E_ADD) return (T)((U)a + (U)b);
    if (OP == E_SUB) return (T)((U)a - (U)b);
    if (OP == E_RSUB) return (T)((U)b - (U)a);
    if (OP == E_MUL) return (T)((U)a * (U)b);
    if (OP == E_DIVC) {
        if (std::is_signed<T>::value && b == (T)-1)
            return (T)((U)0 - (U)a);          // MIN / -1 wraps to MIN
        return a / b;                         // truncates toward zero
    }
    if (OP == E_CONST) return b;
    return a;                                 // E_COPY (type conversion)
}

// dst[r] = a[r] OP (b[r] | k) over the tile.  Operands stored in another type are
// converted into T (mod 2^w); same-type operands are loaded directly.
template <int NT, int ITEMS, typename T, int OP, bool BSLOT>
__device__ __forceinline__ void expr_loop(char *dst, const char *a, int ta, const char *b, int tb, T k)
{
    const int tid = threadIdx.x;
    constexpr int TT = sizeof(T) == 8 ? (std::is_signed<T>::value ? T_I64 : T_U64)
                                      : (std::is_signed<T>::value ? T_I32 : T_U32);
    const bool sa = (ta == TT) || (sizeof(T) == 4 && (ta == T_I32 || ta == T_U32)) ||
                    (sizeof(T) == 8 && (ta == T_I64 || ta == T_U64));
    const bool sb = (tb == TT) || (sizeof(T) == 4 && (tb == T_I32 || tb == T_U32)) ||
                    (sizeof(T) == 8 && (tb == T_I64 || tb == T_U64));
    if (sa && (!BSLOT || sb)) {
#pragma unroll
        for (int i = 0; i < ITEMS; i++) {
            const int r = i * NT + tid;
            const T x = (OP == E_CONST) ? (T)0 : ld_as<T>(a, r);
            const T y = BSLOT ? ld_as<T>(b, r) : k;
            ((T *)dst)[r] = ev<T, OP>(x, y);
        }
    } else {
#pragma unroll
        for (int i = 0; i < ITEMS; i++) {
            const int r = i * NT + tid;
            const T x = (OP == E_CONST) ? (T)0 : (T)ld_ext(a, ta, r);
            const T y = BSLOT ? (T)ld_ext(b, tb, r) : k;
            ((T *)dst)[r] = ev<T, OP>(x, y);
        }
    }
}

// Fused fixed-point factor (plan peephole of MUL over ADD/RSUB with a constant,
// e.g. Q1's price * (100 - disc) and disc_price * (100 + tax), P:223 pattern (e)):
// dst = a * (k +- b), all three of type T, wrapping mod 2^w like the two ops it replaces.
template <int NT, int ITEMS, typename T>
__device__ __forceinline__ void mulaff_loop(char *dst, const char *a, const char *b, T k, bool neg)
{
    typedef typename std::make_unsigned<T>::type U;
    const int tid = threadIdx.x;
    if (neg) {
#pragma unroll
        for (int i = 0; i < ITEMS; i++) {
            const int r = i * NT + tid;
            ((T *)dst)[r] = (T)((U)ld_as<T>(a, r) * ((U)k - (U)ld_as<T>(b, r)));
        }
    } else {
#pragma unroll
        for (int i = 0; i < ITEMS; i++) {
            const int r = i * NT + tid;
            ((T *)dst)[r] = (T)((U)ld_as<T>(a, r) * ((U)k + (U)ld_as<T>(b, r)));
        }
    }
}

#define RW_EXPR_CASES(TT, TCODE)                                                                                  \
    case TCODE * 8 + E_COPY: expr_loop<NT, ITEMS, TT, E_COPY, false>(dst, a, ta, b, tb, (TT)k); return;       \
    case TCODE * 8 + E_CONST: expr_loop<NT, ITEMS, TT, E_CONST, false>(dst, a, ta, b, tb, (TT)k); return;     \
    case TCODE * 8 + E_ADD: expr_loop<NT, ITEMS, TT, E_ADD, false>(dst, a, ta, b, tb, (TT)k); return;         \
    case TCODE * 8 + E_SUB: expr_loop<NT, ITEMS, TT, E_SUB, false>(dst, a, ta, b, tb, (TT)k); return;         \
    case TCODE * 8 + E_MUL: expr_loop<NT, ITEMS, TT, E_MUL, false>(dst, a, ta, b, tb, (TT)k); return;         \
    case TCODE * 8 + E_DIVC: expr_loop<NT, ITEMS, TT, E_DIVC, false>(dst, a, ta, b, tb, (TT)k); return;       \
    case TCODE * 8 + E_RSUB: expr_loop<NT, ITEMS, TT, E_RSUB, false>(dst, a, ta, b, tb, (TT)k); return;       \
    case 64 + TCODE * 8 + E_ADD: expr_loop<NT, ITEMS, TT, E_ADD, true>(dst, a, ta, b, tb, (TT)0); return;       \
    case 64 + TCODE * 8 + E_SUB: expr_loop<NT, ITEMS, TT, E_SUB, true>(dst, a, ta, b, tb, (TT)0); return;       \
    case 64 + TCODE * 8 + E_MUL: expr_loop<NT, ITEMS, TT, E_MUL, true>(dst, a, ta, b, tb, (TT)0); return;       \
    case 64 + TCODE * 8 + E_MULAFF: mulaff_loop<NT, ITEMS, TT>(dst, a, b, (TT)k, (tb & kNegB) != 0); return;

template <int NT, int ITEMS>
__device__ __noinline__ void run_expr(uint32_t code, int ta, int tb, int64_t k, char *dst, const char *a, const char *b)
{
    switch (code) {
        RW_EXPR_CASES(int32_t, T_I32)
        RW_EXPR_CASES(uint32_t, T_U32)
        RW_EXPR_CASES(int64_t, T_I64)
        RW_EXPR_CASES(uint64_t, T_U64)
    }
}

// Run the fused program over one tile (§4.3.1: SELECT / PROJECT in order,
// in the same thread, no synchronisation between thread-dependent operators).
template <int NT, int ITEMS>
__device__ __forceinline__ uint32_t run_ops(const ChainProg &P, int op0, int op1, const char *stage, char *scratch,
                                            uint32_t mask)
{
#pragma unroll 1
    for (int i = op0; i < op1; i++) {
        // fields are read once from the constant bank and passed by value (a reference
        // into kernel-parameter space would turn every field access into a generic load)
        const uint32_t kind = P.ops[i].kind, code = P.ops[i].code;
        const int64_t k = P.ops[i].k;
        const char *a = loc_ptr(P.ops[i].a, stage, scratch);
        const char *b = loc_ptr(P.ops[i].b, stage, scratch);
        if (kind == K_PRED) {
            // inline fast paths for the commonest atoms (32-bit column vs constant);
            // everything else goes through the generic dispatch
            if (code == T_I32 * 8 + C_LT)
                mask = pred_loop<NT, ITEMS, int32_t, C_LT, false>(a, b, (int32_t)k, mask);
            else if (code == T_U32 * 8 + C_LT)
                mask = pred_loop<NT, ITEMS, uint32_t, C_LT, false>(a, b, (uint32_t)k, mask);
            else if (code == T_I32 * 8 + C_LE)
                mask = pred_loop<NT, ITEMS, int32_t, C_LE, false>(a, b, (int32_t)k, mask);
            else
                mask = run_pred<NT, ITEMS>(code, k, a, b, mask);
        }
        else
            run_expr<NT, ITEMS>(code, P.ops[i].ta, P.ops[i].tb, k, (char *)loc_ptr(P.ops[i].dst, stage, scratch), a, b);
    }
    return mask;
}

// ---------------------------------------------------------------------------
// Aggregate terminal (Q1): thread-private int64 partials in smem,
// flushed into 128-bit CTA accumulators before they could overflow (period from
// the plan's interval analysis), CTA accumulators added into global 128-bit
// accumulators with one atomic pair per (group, aggregate) per CTA.
// Partial layout: part[(g * NA + a) * kThreads + tid], a = 0 is the row count.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void atomic_add128(unsigned long long *lo, unsigned long long *hi,
                                              unsigned long long vlo, unsigned long long vhi)
{
    unsigned long long old = atomicAdd(lo, vlo);
    unsigned long long carry = (old + vlo) < old ? 1ull : 0ull;
    unsigned long long h = vhi + carry;
    if (h)
        atomicAdd(hi, h);
}

template <int NT>
__device__ inline void agg_flush(const ChainProg &P, unsigned long long *part, unsigned long long *cta_acc)
{
    const int tid = threadIdx.x;
    const int NA = P.nagg + 1;
    const int n = P.D * NA;
    for (int q = 0; q < n; q++) {
        unsigned long long v = part[q * NT + tid];
        if (v) {
            const int a = q % NA;
            const bool uns = a > 0 && P.agg_unsigned[a - 1];
            unsigned long long hi = (!uns && (long long)v < 0) ? ~0ull : 0ull;
            atomic_add128(&cta_acc[2 * q], &cta_acc[2 * q + 1], v, hi);
            part[q * NT + tid] = 0;
        }
    }
}

// Per-row reference path (used when the partials must be flushed more often than
// every ITEMS rows, i.e. without declared value bounds).
template <int NT, int ITEMS>
__device__ inline void agg_tile_rowwise(const ChainProg &P, const char *stage, const char *scratch, uint32_t mask,
                                        unsigned long long *part, unsigned long long *cta_acc, int64_t &since_flush,
                                        int32_t *err)
{
    const int tid = threadIdx.x;
    const int NA = P.nagg + 1;
#pragma unroll 1
    for (int k = 0; k < ITEMS; k++) {
        if (!((mask >> k) & 1u))
            continue;
        const int r = k * NT + tid;
        int g = 0;
        bool ok = true;
        for (int c = 0; c < P.ngc; c++) {
            const uint64_t code = ld_ext(loc_ptr(P.g_loc[c], stage, scratch), P.g_type[c], r);
            // negative signed codes become huge unsigned values -> out of domain
            if (code >= (uint64_t)P.gdomain[c])
                ok = false;
            g = g * P.gdomain[c] + (int)code;
        }
        if (!ok) {
            atomicAdd(err, 1);
            continue;
        }
        unsigned long long *pg = part + (size_t)g * NA * NT + tid;
        pg[0] += 1ull;
        for (int a = 0; a < P.nagg; a++)
            pg[(a + 1) * NT] += ld_ext(loc_ptr(P.agg_loc[a], stage, scratch), P.agg_type[a], r);
        if (++since_flush >= P.flush_rows) {
            agg_flush<NT>(P, part, cta_acc);
            since_flush = 0;
        }
    }
}

// Row of mask bit k: the scan kernels' k*NT + tid, or (R4) the 4-row vector layout of
// chain4.cuh, ((k/4)*NT + tid)*4 + k%4 (the join expansion's aggregate terminal).
template <int NT, bool R4>
__device__ __forceinline__ int arow(int k)
{
    return R4 ? (((k >> 2) * NT + (int)threadIdx.x) << 2) + (k & 3) : k * NT + (int)threadIdx.x;
}

// Global-atomic terminal (agg_mode 3) for group-bys too large for per-thread
// partials in shared memory: every row adds into the global 128-bit accumulators.
template <int NT, int ITEMS, bool R4 = false>
__device__ inline void agg_tile_global(const ChainProg &P, const char *stage, const char *scratch, uint32_t mask,
                                       unsigned long long *acc, int32_t *err)
{
    const int tid = threadIdx.x;
    const int NA = P.nagg + 1;
#pragma unroll 1
    for (int k = 0; k < ITEMS; k++) {
        if (!((mask >> k) & 1u))
            continue;
        const int r = arow<NT, R4>(k);
        int g = 0;
        bool ok = true;
        for (int c = 0; c < P.ngc; c++) {
            const uint64_t code = ld_ext(loc_ptr(P.g_loc[c], stage, scratch), P.g_type[c], r);
            if (code >= (uint64_t)P.gdomain[c])
                ok = false;
            g = g * P.gdomain[c] + (int)code;
        }
        if (!ok) {
            atomicAdd(err, 1);
            continue;
        }
        unsigned long long *pg = acc + 2 * (size_t)g * NA;
        atomic_add128(&pg[0], &pg[1], 1ull, 0ull);
        for (int a = 0; a < P.nagg; a++) {
            const unsigned long long v = ld_ext(loc_ptr(P.agg_loc[a], stage, scratch), P.agg_type[a], r);
            const unsigned long long hi = (!P.agg_unsigned[a] && (long long)v < 0) ? ~0ull : 0ull;
            atomic_add128(&pg[2 * (a + 1)], &pg[2 * (a + 1) + 1], v, hi);
        }
    }
}

constexpr int kAggUnroll = 8;

// Tile-wise aggregate terminal: group codes of the thread's ITEMS rows computed
// column by column (type switch hoisted out of the row loop), then each aggregate
// column added into the thread-private partials; the aggregate loop is unrolled so
// the independent read-modify-write chains of different aggregates overlap.
template <int NT, int ITEMS>
__device__ inline void agg_tile(const ChainProg &P, const char *stage, const char *scratch, uint32_t mask,
                                unsigned long long *part, unsigned long long *cta_acc, int64_t &since_flush,
                                int32_t *err)
{
    if (P.flush_rows < ITEMS || P.nagg > kAggUnroll) {
        agg_tile_rowwise<NT, ITEMS>(P, stage, scratch, mask, part, cta_acc, since_flush, err);
        return;
    }
    const int tid = threadIdx.x;
    const int NA = P.nagg + 1;
    uint32_t g[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++)
        g[k] = 0;
    uint32_t ok = mask;
    for (int c = 0; c < P.ngc; c++) {
        const char *b = loc_ptr(P.g_loc[c], stage, scratch);
        const uint32_t dom = (uint32_t)P.gdomain[c];
        switch (P.g_type[c]) {
        case T_U8:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint32_t v = ((const uint8_t *)b)[k * NT + tid];
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + v;
            }
            break;
        case T_I32:
        case T_U32:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint32_t v = ((const uint32_t *)b)[k * NT + tid];   // negative i32 -> huge
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + v;
            }
            break;
        default:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint64_t v = ((const uint64_t *)b)[k * NT + tid];
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + (uint32_t)v;
            }
            break;
        }
    }
    if (ok != mask)
        atomicAdd(err, __popc(mask & ~ok));
    const int rows = __popc(ok);
    if (since_flush + rows > P.flush_rows) {
        agg_flush<NT>(P, part, cta_acc);
        since_flush = 0;
    }
    since_flush += rows;
    const uint32_t stride = (uint32_t)NA * NT;
#pragma unroll
    for (int k = 0; k < ITEMS; k++)
        if ((ok >> k) & 1u)
            part[g[k] * stride + tid] += 1ull;
#pragma unroll
    for (int a = 0; a < kAggUnroll; a++) {
        if (a < P.nagg) {
            const char *b = loc_ptr(P.agg_loc[a], stage, scratch);
            unsigned long long *pa = part + (a + 1) * NT + tid;
            const int t = P.agg_type[a];
            if (t == T_I64 || t == T_U64) {
#pragma unroll
                for (int k = 0; k < ITEMS; k++)
                    if ((ok >> k) & 1u)
                        pa[g[k] * stride] += ((const uint64_t *)b)[k * NT + tid];
            } else {
#pragma unroll
                for (int k = 0; k < ITEMS; k++)
                    if ((ok >> k) & 1u)
                        pa[g[k] * stride] += ld_ext(b, t, k * NT + tid);
            }
        }
    }
}

// Register terminal (agg_mode 2) for small group-bys (D <= kRegD groups, nagg <=
// kRegA sums, e.g. Q1's 6 x 5): every compute thread keeps its int64 partials of
// all (group, sum) pairs in registers and adds a row into the pairs of its group
// with predicated adds (one-hot over the D groups, no shared-memory traffic and no
// dependent read-modify-write chains).  The plan picks this mode only when the
// interval analysis allows >= 2^16 rows per thread between flushes; a flush adds
// the registers into the CTA's 128-bit accumulators.
struct RegAgg {
    uint64_t s[kRegD][kRegA];
    uint32_t n[kRegD][kRegA];      // narrow sums (a < P.agg_narrow): 32-bit partials
    uint32_t c[kRegD];
};

__device__ __forceinline__ void reg_agg_zero(RegAgg &R)
{
#pragma unroll
    for (int d = 0; d < kRegD; d++) {
        R.c[d] = 0;
#pragma unroll
        for (int a = 0; a < kRegA; a++) {
            R.s[d][a] = 0;
            R.n[d][a] = 0;
        }
    }
}

// adds the registers into 128-bit accumulators acc[2*(g*NA + a)] (shared, atomically)
__device__ inline void reg_agg_flush(const ChainProg &P, RegAgg &R, unsigned long long *acc)
{
    const int NA = P.nagg + 1;
#pragma unroll
    for (int d = 0; d < kRegD; d++) {
        if (d < P.D && R.c[d]) {
            atomic_add128(&acc[2 * (d * NA)], &acc[2 * (d * NA) + 1], R.c[d], 0ull);
#pragma unroll
            for (int a = 0; a < kRegA; a++) {
                if (a < P.nagg) {
                    const bool nar = a < P.agg_narrow;
                    const unsigned long long v = nar ? (unsigned long long)R.n[d][a] : R.s[d][a];
                    const unsigned long long hi = (!nar && !P.agg_unsigned[a] && (long long)v < 0) ? ~0ull : 0ull;
                    atomic_add128(&acc[2 * (d * NA + 1 + a)], &acc[2 * (d * NA + 1 + a) + 1], v, hi);
                }
            }
        }
    }
    reg_agg_zero(R);
}

// stores the registers as thread-private partials part[(g*NA + a)*NT + tid] for agg_combine
template <int NT>
__device__ inline void reg_agg_store(const ChainProg &P, const RegAgg &R, unsigned long long *part)
{
    const int NA = P.nagg + 1, tid = threadIdx.x;
#pragma unroll
    for (int d = 0; d < kRegD; d++) {
        if (d < P.D) {
            part[(d * NA) * NT + tid] = R.c[d];
#pragma unroll
            for (int a = 0; a < kRegA; a++)
                if (a < P.nagg)
                    part[(d * NA + 1 + a) * NT + tid] = a < P.agg_narrow ? (unsigned long long)R.n[d][a] : R.s[d][a];
        }
    }
}

// End of the register terminal: every (group, sum) partial is reduced across the
// warp exactly in 128 bits (shuffles), then lane 0 adds the warp's total into the
// CTA's 128-bit accumulators (one shared atomic pair per warp, not per thread).
__device__ __forceinline__ void warp_sum128(unsigned long long &lo, unsigned long long &hi)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long l2 = __shfl_xor_sync(0xffffffffu, lo, o);
        const unsigned long long h2 = __shfl_xor_sync(0xffffffffu, hi, o);
        const unsigned long long nl = lo + l2;
        hi = hi + h2 + (nl < lo ? 1ull : 0ull);
        lo = nl;
    }
}

__device__ inline void reg_agg_reduce_warp(const ChainProg &P, RegAgg &R, unsigned long long *acc)
{
    const int NA = P.nagg + 1;
    const bool lane0 = (threadIdx.x & 31) == 0;
#pragma unroll
    for (int d = 0; d < kRegD; d++) {
        if (d < P.D) {
            unsigned long long lo = R.c[d], hi = 0;
            warp_sum128(lo, hi);
            if (lane0 && (lo | hi))
                atomic_add128(&acc[2 * (d * NA)], &acc[2 * (d * NA) + 1], lo, hi);
#pragma unroll
            for (int a = 0; a < kRegA; a++) {
                if (a < P.nagg) {
                    const bool nar = a < P.agg_narrow;
                    unsigned long long v = nar ? (unsigned long long)R.n[d][a] : R.s[d][a];
                    unsigned long long h = (!nar && !P.agg_unsigned[a] && (long long)v < 0) ? ~0ull : 0ull;
                    warp_sum128(v, h);
                    if (lane0 && (v | h))
                        atomic_add128(&acc[2 * (d * NA + 1 + a)], &acc[2 * (d * NA + 1 + a) + 1], v, h);
                }
            }
        }
    }
    reg_agg_zero(R);
}

// Row loop of the register terminal: NAGG sums (W64: every sum column is 64-bit, so
// no per-row type dispatch); the one-hot over the groups becomes a jump to the
// row's group, whose partials take predicated-free adds.
// Narrow sums (a < NN) accumulate in 32-bit partials whose flush period comes from the
// caller-declared bounds; the values of the aggregated rows are OR-ed into `orv`, so that
// a value outside [0, 2^narrow_bits) is reported (err[2]) instead of silently wrapping a
// partial.
template <int NT, int ITEMS, int NAGG, bool W64, int NN = 0, bool R4 = false>
__device__ __forceinline__ void agg_rows_reg(const char *const *ab, const int *at, const uint32_t *g, uint32_t ok,
                                             RegAgg &R, uint64_t &orv)
{
    const int tid = threadIdx.x;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint32_t gk = ((ok >> k) & 1u) ? g[k] : 0xffffffffu;   // failing rows match no group
        const int r = arow<NT, R4>(k);
        uint64_t v[kRegA];
#pragma unroll
        for (int a = 0; a < kRegA; a++)
            v[a] = a < NAGG ? (W64 ? ((const uint64_t *)ab[a])[r] : ld_ext(ab[a], at[a], r)) : 0ull;
#pragma unroll
        for (int a = 0; a < NN; a++)
            if ((ok >> k) & 1u)   // aggregated rows only (a ragged tile's tail holds stale data)
                orv |= v[a];
#pragma unroll
        for (int d = 0; d < kRegD; d++) {
            if (gk == (uint32_t)d) {
                R.c[d] += 1u;
#pragma unroll
                for (int a = 0; a < NAGG; a++) {
                    if (a < NN)
                        R.n[d][a] += (uint32_t)v[a];
                    else
                        R.s[d][a] += v[a];
                }
            }
        }
    }
}

template <int NT, int ITEMS, bool R4 = false>
__device__ inline void agg_tile_reg(const ChainProg &P, const char *stage, const char *scratch, uint32_t mask,
                                    RegAgg &R, unsigned long long *cta_acc, int64_t &since_flush, int32_t *err)
{
    const int tid = threadIdx.x;
    uint32_t g[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++)
        g[k] = 0;
    uint32_t ok = mask;
    for (int c = 0; c < P.ngc; c++) {
        const char *b = loc_ptr(P.g_loc[c], stage, scratch);
        const uint32_t dom = (uint32_t)P.gdomain[c];
        switch (P.g_type[c]) {
        case T_U8:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint32_t v = ((const uint8_t *)b)[arow<NT, R4>(k)];
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + v;
            }
            break;
        case T_I32:
        case T_U32:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint32_t v = ((const uint32_t *)b)[arow<NT, R4>(k)];   // negative i32 -> huge
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + v;
            }
            break;
        default:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint64_t v = ((const uint64_t *)b)[arow<NT, R4>(k)];
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + (uint32_t)v;
            }
            break;
        }
    }
    if (ok != mask)
        atomicAdd(err, __popc(mask & ~ok));
    const int rows = __popc(ok);
    if (since_flush + rows > P.flush_rows) {
        reg_agg_flush(P, R, cta_acc);
        since_flush = 0;
    }
    since_flush += rows;
    const char *ab[kRegA];
    int at[kRegA];
    bool w64 = true;
#pragma unroll
    for (int a = 0; a < kRegA; a++) {
        ab[a] = a < P.nagg ? loc_ptr(P.agg_loc[a], stage, scratch) : nullptr;
        at[a] = a < P.nagg ? P.agg_type[a] : T_U64;
        if (a < P.nagg && !(at[a] == T_I64 || at[a] == T_U64))
            w64 = false;
    }
    // the sum count and the all-64-bit case are compile-time in the row loop
    uint64_t orv = 0;
    if (NT == kNarrowNT) {
        // the 576-thread instance is specialised (host-selected) for 5 all-64-bit sums of
        // which the first 2 are narrow: only this row loop is compiled into it, which is
        // what lets 18 compute warps fit the register file
        agg_rows_reg<NT, ITEMS, 5, true, 2, R4>(ab, at, g, ok, R, orv);
    } else if (w64 && P.agg_narrow) {
        switch (P.nagg * 4 + P.agg_narrow) {
        case 3 * 4 + 1: agg_rows_reg<NT, ITEMS, 3, true, 1, R4>(ab, at, g, ok, R, orv); break;
        case 3 * 4 + 2: agg_rows_reg<NT, ITEMS, 3, true, 2, R4>(ab, at, g, ok, R, orv); break;
        case 4 * 4 + 1: agg_rows_reg<NT, ITEMS, 4, true, 1, R4>(ab, at, g, ok, R, orv); break;
        case 4 * 4 + 2: agg_rows_reg<NT, ITEMS, 4, true, 2, R4>(ab, at, g, ok, R, orv); break;
        case 5 * 4 + 1: agg_rows_reg<NT, ITEMS, 5, true, 1, R4>(ab, at, g, ok, R, orv); break;
        default: agg_rows_reg<NT, ITEMS, 5, true, 2, R4>(ab, at, g, ok, R, orv); break;
        }
    } else if (w64) {
        switch (P.nagg) {
        case 0: agg_rows_reg<NT, ITEMS, 0, true, 0, R4>(ab, at, g, ok, R, orv); break;
        case 1: agg_rows_reg<NT, ITEMS, 1, true, 0, R4>(ab, at, g, ok, R, orv); break;
        case 2: agg_rows_reg<NT, ITEMS, 2, true, 0, R4>(ab, at, g, ok, R, orv); break;
        case 3: agg_rows_reg<NT, ITEMS, 3, true, 0, R4>(ab, at, g, ok, R, orv); break;
        case 4: agg_rows_reg<NT, ITEMS, 4, true, 0, R4>(ab, at, g, ok, R, orv); break;
        default: agg_rows_reg<NT, ITEMS, kRegA, true, 0, R4>(ab, at, g, ok, R, orv); break;
        }
    } else {
        agg_rows_reg<NT, ITEMS, kRegA, false, 0, R4>(ab, at, g, ok, R, orv);
    }
    // a narrow value outside its declared bounds: report (err[2]) rather than wrap
    if (orv >> P.narrow_bits)
        atomicAdd(err + 2, 1);
}

// Fused row path of the kNarrowNT instance for the TPC-H Q1 program shape (host-checked,
// ChainProg::q1fused, pattern (e) of Fig. 14): ops = [SELECT i32 column vs
// constant, d = a * (k1 -/+ b), c = d * (k2 -/+ e)] and sums = [2 narrow stage columns,
// 1 wide stage column, d, c].  The same arithmetic as the interpreter (wrap mod 2^64,
// reading A8), evaluated per row in registers: the computed columns never touch shared
// memory and there is no per-op dispatch (the paper generates this code per fused group,
// P:177-179; here it is compiled ahead of time for this shape).
template <int NT, int ITEMS>
__device__ inline void agg_tile_q1(const ChainProg &P, const char *stage, uint32_t mask, RegAgg &R,
                                   unsigned long long *cta_acc, int64_t &since_flush, int32_t *err)
{
    const int tid = threadIdx.x;
    // SELECT atom: the common comparisons inline, the rest through the generic dispatch
    const uint32_t pcode = P.ops[0].code;
    const int64_t pk = P.ops[0].k;
    const char *pa = stage + P.ops[0].a;
    uint32_t ok;
    if (pcode == T_I32 * 8 + C_LE)
        ok = pred_loop<NT, ITEMS, int32_t, C_LE, false>(pa, nullptr, (int32_t)pk, mask);
    else if (pcode == T_I32 * 8 + C_LT)
        ok = pred_loop<NT, ITEMS, int32_t, C_LT, false>(pa, nullptr, (int32_t)pk, mask);
    else
        ok = run_pred<NT, ITEMS>(pcode, pk, pa, nullptr, mask);
    // group codes (first group column slowest), out-of-domain rows counted
    uint32_t g[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++)
        g[k] = 0;
    const uint32_t sel = ok;
    for (int c = 0; c < P.ngc; c++) {
        const char *b = stage + P.g_loc[c];
        const uint32_t dom = (uint32_t)P.gdomain[c];
        switch (P.g_type[c]) {
        case T_U8:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint32_t v = ((const uint8_t *)b)[k * NT + tid];
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + v;
            }
            break;
        case T_I32:
        case T_U32:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint32_t v = ((const uint32_t *)b)[k * NT + tid];
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + v;
            }
            break;
        default:
#pragma unroll
            for (int k = 0; k < ITEMS; k++) {
                const uint64_t v = ((const uint64_t *)b)[k * NT + tid];
                if (v >= dom) ok &= ~(1u << k);
                g[k] = g[k] * dom + (uint32_t)v;
            }
            break;
        }
    }
    if (ok != sel)
        atomicAdd(err, __popc(sel & ~ok));
    const int rows = __popc(ok);
    if (since_flush + rows > P.flush_rows) {
        reg_agg_flush(P, R, cta_acc);
        since_flush = 0;
    }
    since_flush += rows;
    const uint64_t *xa = (const uint64_t *)(stage + P.ops[1].a);   // e.g. price
    const uint64_t *xb = (const uint64_t *)(stage + P.ops[1].b);   // e.g. disc
    const uint64_t *xe = (const uint64_t *)(stage + P.ops[2].b);   // e.g. tax
    const uint64_t k1 = (uint64_t)P.ops[1].k, k2 = (uint64_t)P.ops[2].k;
    const bool n1 = (P.ops[1].tb & kNegB) != 0, n2 = (P.ops[2].tb & kNegB) != 0;
    const uint64_t *s0 = (const uint64_t *)(stage + P.agg_loc[0]);
    const uint64_t *s1 = (const uint64_t *)(stage + P.agg_loc[1]);
    const uint64_t *s2 = (const uint64_t *)(stage + P.agg_loc[2]);
    uint64_t orv = 0;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const bool on = (ok >> k) & 1u;
        const uint32_t gk = on ? g[k] : 0xffffffffu;   // failing rows match no group
        const int r = k * NT + tid;
        const uint64_t b = xb[r], e = xe[r];
        const uint64_t d = xa[r] * (n1 ? k1 - b : k1 + b);
        const uint64_t c = d * (n2 ? k2 - e : k2 + e);
        const uint64_t v0 = s0[r], v1 = s1[r], v2 = s2[r];
        if (on)
            orv |= v0 | v1;
#pragma unroll
        for (int dd = 0; dd < kRegD; dd++) {
            if (gk == (uint32_t)dd) {
                R.c[dd] += 1u;
                R.n[dd][0] += (uint32_t)v0;
                R.n[dd][1] += (uint32_t)v1;
                R.s[dd][2] += v2;
                R.s[dd][3] += d;
                R.s[dd][4] += c;
            }
        }
    }
    if (orv >> P.narrow_bits)
        atomicAdd(err + 2, 1);
}

// End-of-kernel combine of the thread-private partials: one thread per (group,
// aggregate) slot sums the NT partials exactly in 128 bits (no shared atomics, whose
// 64-bit form is a CAS loop on sm_100), then adds the slot into cta_acc.
template <int NT>
__device__ inline void agg_combine(const ChainProg &P, unsigned long long *part, unsigned long long *cta_acc,
                                   int nthreads)
{
    const int NA = P.nagg + 1;
    for (int q = threadIdx.x; q < P.D * NA; q += nthreads) {
        const int a = q % NA;
        const bool uns = a > 0 && P.agg_unsigned[a - 1];
        unsigned long long lo = cta_acc[2 * q], hi = cta_acc[2 * q + 1];
        for (int t = 0; t < NT; t++) {
            const unsigned long long v = part[q * NT + t];
            const unsigned long long vh = (!uns && (long long)v < 0) ? ~0ull : 0ull;
            const unsigned long long nlo = lo + v;
            hi += vh + (nlo < lo ? 1ull : 0ull);
            lo = nlo;
        }
        cta_acc[2 * q] = lo;
        cta_acc[2 * q + 1] = hi;
    }
}

}  // namespace rw
