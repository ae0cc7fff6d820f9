// chain.cuh — device side of a fused group: the per-tile micro-op interpreter
// (SELECT atoms, PROJECT / arithmetic), warp-ballot compaction, block scan,
// decoupled look-back, compacted store, and the group-by aggregate terminal.
//
// Tile layout: T = kThreads * ITEMS rows; thread `tid` owns rows k*kThreads+tid
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

__device__ inline uint64_t lookback_warp(uint64_t *status, int64_t tile, uint64_t agg, uint32_t epoch)
{
    const int lane = threadIdx.x & 31;
    const uint64_t tag = (uint64_t)epoch << 48;
    if (tile == 0) {
        if (lane == 0)
            st_relaxed_u64(&status[0], tag | (2ull << 46) | agg);
        return 0;
    }
    if (lane == 0)
        st_relaxed_u64(&status[tile], tag | (1ull << 46) | agg);
    uint64_t excl = 0;
    int64_t j = tile - 1;
    while (true) {
        int64_t idx = j - lane;
        uint32_t flag = 2;
        uint64_t val = 0;
        if (idx >= 0) {
            uint64_t w;
            do {
                w = ld_relaxed_u64(&status[idx]);
                flag = ((uint32_t)(w >> 48) == epoch) ? (uint32_t)(w >> 46) & 3u : 0u;
            } while (flag == 0);
            val = w & kValMask;
        }
        uint32_t pmask = __ballot_sync(0xffffffffu, flag == 2);
        if (pmask) {
            int first = __ffs(pmask) - 1;          // nearest predecessor holding an inclusive prefix
            excl += warp_sum_u64(lane <= first ? val : 0);
            break;
        }
        excl += warp_sum_u64(val);
        j -= 32;
    }
    if (lane == 0)
        st_relaxed_u64(&status[tile], tag | (2ull << 46) | (excl + agg));
    return excl;
}

// ---------------------------------------------------------------------------
// Slot access
// ---------------------------------------------------------------------------
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
template <int ITEMS, typename T, int CMP>
__device__ __forceinline__ uint32_t pred_loop(const char *a, const char *b, T k, bool bslot, uint32_t mask)
{
    const int tid = threadIdx.x;
    const T *pa = (const T *)a;
    const T *pb = (const T *)b;
#pragma unroll
    for (int i = 0; i < ITEMS; i++) {
        T x = pa[i * kThreads + tid];
        T y = bslot ? pb[i * kThreads + tid] : k;
        if (!cmpv<T, CMP>(x, y))
            mask &= ~(1u << i);
    }
    return mask;
}

template <int ITEMS, typename T>
__device__ __forceinline__ uint32_t pred_t(int cmp, const char *a, const char *b, int64_t k, bool bslot, uint32_t mask)
{
    T kk = (T)k;
    switch (cmp) {
    case C_LT: return pred_loop<ITEMS, T, C_LT>(a, b, kk, bslot, mask);
    case C_LE: return pred_loop<ITEMS, T, C_LE>(a, b, kk, bslot, mask);
    case C_GT: return pred_loop<ITEMS, T, C_GT>(a, b, kk, bslot, mask);
    case C_GE: return pred_loop<ITEMS, T, C_GE>(a, b, kk, bslot, mask);
    case C_EQ: return pred_loop<ITEMS, T, C_EQ>(a, b, kk, bslot, mask);
    default: return pred_loop<ITEMS, T, C_NE>(a, b, kk, bslot, mask);
    }
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

template <int ITEMS, typename T, int OP>
__device__ __forceinline__ void expr_loop(char *dst, const char *a, int ta, const char *b, int tb, bool bslot, T k)
{
    const int tid = threadIdx.x;
#pragma unroll
    for (int i = 0; i < ITEMS; i++) {
        const int r = i * kThreads + tid;
        T x = (OP == E_CONST) ? (T)0 : (T)ld_ext(a, ta, r);
        T y = bslot ? (T)ld_ext(b, tb, r) : k;
        ((T *)dst)[r] = ev<T, OP>(x, y);
    }
}

template <int ITEMS, typename T>
__device__ __forceinline__ void expr_t(const DevOp &o, char *dst, const char *a, int ta, const char *b, int tb)
{
    const bool bs = o.b_is_slot;
    const T k = (T)o.k;
    switch (o.op) {
    case E_COPY: expr_loop<ITEMS, T, E_COPY>(dst, a, ta, b, tb, false, k); break;
    case E_CONST: expr_loop<ITEMS, T, E_CONST>(dst, a, ta, b, tb, false, k); break;
    case E_ADD: expr_loop<ITEMS, T, E_ADD>(dst, a, ta, b, tb, bs, k); break;
    case E_SUB: expr_loop<ITEMS, T, E_SUB>(dst, a, ta, b, tb, bs, k); break;
    case E_MUL: expr_loop<ITEMS, T, E_MUL>(dst, a, ta, b, tb, bs, k); break;
    case E_RSUB: expr_loop<ITEMS, T, E_RSUB>(dst, a, ta, b, tb, false, k); break;
    default: expr_loop<ITEMS, T, E_DIVC>(dst, a, ta, b, tb, false, k); break;
    }
}

// Run the fused program over one tile (§4.3.1: SELECT / PROJECT in order,
// in the same thread, no synchronisation between thread-dependent operators).
template <int ITEMS>
__device__ __forceinline__ uint32_t run_ops(const ChainProg &P, const char *stage, char *scratch, uint32_t mask)
{
    for (int i = 0; i < P.nops; i++) {
        const DevOp &o = P.ops[i];
        const char *a = o.a >= 0 ? slot_ptr(P, o.a, stage, scratch) : nullptr;
        const char *b = (o.b_is_slot && o.b >= 0) ? slot_ptr(P, o.b, stage, scratch) : nullptr;
        if (o.kind == K_PRED) {
            switch (o.type) {
            case T_I32: mask = pred_t<ITEMS, int32_t>(o.op, a, b, o.k, o.b_is_slot, mask); break;
            case T_U32: mask = pred_t<ITEMS, uint32_t>(o.op, a, b, o.k, o.b_is_slot, mask); break;
            case T_I64: mask = pred_t<ITEMS, int64_t>(o.op, a, b, o.k, o.b_is_slot, mask); break;
            case T_U64: mask = pred_t<ITEMS, uint64_t>(o.op, a, b, o.k, o.b_is_slot, mask); break;
            default: mask = pred_t<ITEMS, uint8_t>(o.op, a, b, o.k, o.b_is_slot, mask); break;
            }
        } else {
            char *dst = (char *)slot_ptr(P, o.dst, stage, scratch);
            const int ta = o.a >= 0 ? P.slot[o.a].type : T_I64;
            const int tb = (o.b_is_slot && o.b >= 0) ? P.slot[o.b].type : T_I64;
            switch (o.type) {
            case T_I32: expr_t<ITEMS, int32_t>(o, dst, a, ta, b, tb); break;
            case T_U32: expr_t<ITEMS, uint32_t>(o, dst, a, ta, b, tb); break;
            case T_I64: expr_t<ITEMS, int64_t>(o, dst, a, ta, b, tb); break;
            default: expr_t<ITEMS, uint64_t>(o, dst, a, ta, b, tb); break;
            }
        }
    }
    return mask;
}

// ---------------------------------------------------------------------------
// Materialising terminal: ballot compaction + block scan + look-back + store.
// ---------------------------------------------------------------------------
template <int ITEMS>
struct EmitSmem {
    uint32_t cnt[ITEMS * kWarps];   // survivors per (item k, warp), then exclusive prefixes
    int64_t tile_off;
};

template <int ITEMS, typename T>
__device__ __forceinline__ void store_col(T *dst, const T *src, uint32_t mask, const uint32_t *bal,
                                          const uint32_t *pre, int64_t base, int64_t cap)
{
    const int tid = threadIdx.x, warp = tid >> 5;
    const uint32_t lt = lanemask_lt();
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        if ((mask >> k) & 1u) {
            int64_t pos = base + pre[k * kWarps + warp] + __popc(bal[k] & lt);
            if (pos < cap)
                dst[pos] = src[k * kThreads + tid];
        }
    }
}

template <int ITEMS>
__device__ inline void emit_tile(const ChainProg &P, const char *stage, const char *scratch, uint32_t mask,
                                 int64_t tile, int64_t ntiles, const TileLaunch &L, EmitSmem<ITEMS> *es)
{
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    uint32_t bal[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        bal[k] = __ballot_sync(0xffffffffu, (mask >> k) & 1u);
        if (lane == 0)
            es->cnt[k * kWarps + warp] = __popc(bal[k]);
    }
    __syncthreads();
    if (warp == 0) {
        constexpr int NV = ITEMS * kWarps;
        constexpr int PER = (NV + 31) / 32;
        uint32_t v[PER];
        uint32_t s = 0;
#pragma unroll
        for (int q = 0; q < PER; q++) {
            int idx = lane * PER + q;
            v[q] = idx < NV ? es->cnt[idx] : 0;
            s += v[q];
        }
        uint32_t inc = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o)
                inc += y;
        }
        uint32_t total = __shfl_sync(0xffffffffu, inc, 31);
        uint32_t run = inc - s;
#pragma unroll
        for (int q = 0; q < PER; q++) {
            int idx = lane * PER + q;
            if (idx < NV)
                es->cnt[idx] = run;
            run += v[q];
        }
        uint64_t excl = lookback_warp(L.status, tile, total, L.epoch);
        if (lane == 0) {
            es->tile_off = (int64_t)excl;
            if (tile == ntiles - 1)
                *L.n_dev = (int64_t)(excl + total);
        }
    }
    __syncthreads();
    const int64_t base = es->tile_off;
    for (int j = 0; j < P.nout; j++) {
        const int s = P.out_slot[j];
        const char *src = slot_ptr(P, s, stage, scratch);
        switch (type_width(P.slot[s].type)) {
        case 1: store_col<ITEMS, uint8_t>((uint8_t *)P.out_ptr[j], (const uint8_t *)src, mask, bal, es->cnt, base, P.out_capacity); break;
        case 4: store_col<ITEMS, uint32_t>((uint32_t *)P.out_ptr[j], (const uint32_t *)src, mask, bal, es->cnt, base, P.out_capacity); break;
        default: store_col<ITEMS, uint64_t>((uint64_t *)P.out_ptr[j], (const uint64_t *)src, mask, bal, es->cnt, base, P.out_capacity); break;
        }
    }
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

__device__ inline void agg_flush(const ChainProg &P, unsigned long long *part, unsigned long long *cta_acc)
{
    const int tid = threadIdx.x;
    const int NA = P.nagg + 1;
    const int n = P.D * NA;
    for (int q = 0; q < n; q++) {
        unsigned long long v = part[q * kThreads + tid];
        if (v) {
            const int a = q % NA;
            const bool uns = a > 0 && P.agg_unsigned[a - 1];
            unsigned long long hi = (!uns && (long long)v < 0) ? ~0ull : 0ull;
            atomic_add128(&cta_acc[2 * q], &cta_acc[2 * q + 1], v, hi);
            part[q * kThreads + tid] = 0;
        }
    }
}

template <int ITEMS>
__device__ inline void agg_tile(const ChainProg &P, const char *stage, const char *scratch, uint32_t mask,
                                unsigned long long *part, unsigned long long *cta_acc, int64_t &since_flush,
                                int32_t *err)
{
    const int tid = threadIdx.x;
    const int NA = P.nagg + 1;
#pragma unroll 1
    for (int k = 0; k < ITEMS; k++) {
        if (!((mask >> k) & 1u))
            continue;
        const int r = k * kThreads + tid;
        int g = 0;
        bool ok = true;
        for (int c = 0; c < P.ngc; c++) {
            const int s = P.gslot[c];
            const int t = P.slot[s].type;
            uint64_t code = ld_ext(slot_ptr(P, s, stage, scratch), t, r);
            // negative signed codes become huge unsigned values -> out of domain
            if (code >= (uint64_t)P.gdomain[c])
                ok = false;
            g = g * P.gdomain[c] + (int)code;
        }
        if (!ok) {
            atomicAdd(err, 1);
            continue;
        }
        unsigned long long *pg = part + (size_t)g * NA * kThreads + tid;
        pg[0] += 1ull;
        for (int a = 0; a < P.nagg; a++) {
            const int s = P.agg_slot[a];
            pg[(a + 1) * kThreads] += ld_ext(slot_ptr(P, s, stage, scratch), P.slot[s].type, r);
        }
        if (++since_flush >= P.flush_rows) {
            agg_flush(P, part, cta_acc);
            since_flush = 0;
        }
    }
}

}  // namespace rw
