// chain4.cuh — the fused-group micro-op interpreter over 4-row vectors.
//
// Tile layout of the emitting scan kernel (scan_emit.cu): thread `tid` owns G groups
// of 4 consecutive rows, group g = rows (g*NT + tid)*4 .. +3, so every slot access is
// one 16-byte shared-memory vector per 4 rows of a 4-byte column (LDS.128 / STS.128;
// two for 8-byte columns, one 32-bit access for byte columns) and a warp's 32 lanes
// cover 128 consecutive rows.  Bit g*4+q of the per-thread `mask` is row
// (g*NT + tid)*4 + q (§5.1.1: the filters of a fused group AND-ed into one
// `match` value per tuple).  Semantics are those of chain.cuh (readings A4, A8).
#pragma once
#include "chain.cuh"

namespace rw {

template <typename T>
struct V4 {
    T v[4];
};

// 4 consecutive rows of a column starting at row r0 (r0 % 4 == 0; slot bases are
// 128-byte aligned, so every access below is naturally aligned)
template <typename T>
__device__ __forceinline__ V4<T> ld4(const char *base, int r0)
{
    V4<T> o;
    if constexpr (sizeof(T) == 4) {
        const uint4 u = *(const uint4 *)(base + (size_t)r0 * 4);
        o.v[0] = (T)u.x; o.v[1] = (T)u.y; o.v[2] = (T)u.z; o.v[3] = (T)u.w;
    } else if constexpr (sizeof(T) == 8) {
        const ulonglong2 a = *(const ulonglong2 *)(base + (size_t)r0 * 8);
        const ulonglong2 b = *(const ulonglong2 *)(base + (size_t)r0 * 8 + 16);
        o.v[0] = (T)a.x; o.v[1] = (T)a.y; o.v[2] = (T)b.x; o.v[3] = (T)b.y;
    } else {
        const uint32_t u = *(const uint32_t *)(base + r0);
#pragma unroll
        for (int q = 0; q < 4; q++)
            o.v[q] = (T)((u >> (8 * q)) & 0xffu);
    }
    return o;
}

template <typename T>
__device__ __forceinline__ void st4(char *base, int r0, const V4<T> &o)
{
    if constexpr (sizeof(T) == 4) {
        *(uint4 *)(base + (size_t)r0 * 4) = make_uint4((uint32_t)o.v[0], (uint32_t)o.v[1], (uint32_t)o.v[2], (uint32_t)o.v[3]);
    } else if constexpr (sizeof(T) == 8) {
        *(ulonglong2 *)(base + (size_t)r0 * 8) = make_ulonglong2((uint64_t)o.v[0], (uint64_t)o.v[1]);
        *(ulonglong2 *)(base + (size_t)r0 * 8 + 16) = make_ulonglong2((uint64_t)o.v[2], (uint64_t)o.v[3]);
    } else {
        *(uint32_t *)(base + r0) = (uint32_t)(uint8_t)o.v[0] | ((uint32_t)(uint8_t)o.v[1] << 8) |
                                   ((uint32_t)(uint8_t)o.v[2] << 16) | ((uint32_t)(uint8_t)o.v[3] << 24);
    }
}

// 4 rows of a slot of any type, sign/zero-extended to 64 bits (value mod 2^64)
__device__ __forceinline__ V4<uint64_t> ld4_ext(const char *base, int type, int r0)
{
    V4<uint64_t> o;
    switch (type) {
    case T_I32: { V4<int32_t> x = ld4<int32_t>(base, r0); for (int q = 0; q < 4; q++) o.v[q] = (uint64_t)(int64_t)x.v[q]; break; }
    case T_U32: { V4<uint32_t> x = ld4<uint32_t>(base, r0); for (int q = 0; q < 4; q++) o.v[q] = x.v[q]; break; }
    case T_U8: { V4<uint8_t> x = ld4<uint8_t>(base, r0); for (int q = 0; q < 4; q++) o.v[q] = x.v[q]; break; }
    default: o = ld4<uint64_t>(base, r0); break;
    }
    return o;
}

// (threadIdx.x % NT: the emitting scan kernel may run several teams of NT compute
// threads, each on its own tiles; every other kernel's compute threads are [0, NT))
template <int NT>
__device__ __forceinline__ int row4(int g) { return (g * NT + (int)(threadIdx.x % NT)) * 4; }

// SELECT atom over the thread's G x 4 rows: clears the bits of rows failing `a CMP b`
template <int NT, int G, typename T, int CMP, bool BSLOT>
__device__ __forceinline__ uint32_t pred4(const char *a, const char *b, T k, uint32_t mask)
{
    uint32_t keep = 0;
#pragma unroll
    for (int g = 0; g < G; g++) {
        const int r0 = row4<NT>(g);
        const V4<T> x = ld4<T>(a, r0);
        V4<T> y;
        if (BSLOT) y = ld4<T>(b, r0);
#pragma unroll
        for (int q = 0; q < 4; q++)
            keep |= (uint32_t)cmpv<T, CMP>(x.v[q], BSLOT ? y.v[q] : k) << (g * 4 + q);
    }
    return mask & keep;
}

#define RW_PRED4_CASES(TT, TCODE)                                                                       \
    case TCODE * 8 + C_LT: return pred4<NT, G, TT, C_LT, false>(a, b, (TT)k, mask);                     \
    case TCODE * 8 + C_LE: return pred4<NT, G, TT, C_LE, false>(a, b, (TT)k, mask);                     \
    case TCODE * 8 + C_GT: return pred4<NT, G, TT, C_GT, false>(a, b, (TT)k, mask);                     \
    case TCODE * 8 + C_GE: return pred4<NT, G, TT, C_GE, false>(a, b, (TT)k, mask);                     \
    case TCODE * 8 + C_EQ: return pred4<NT, G, TT, C_EQ, false>(a, b, (TT)k, mask);                     \
    case TCODE * 8 + C_NE: return pred4<NT, G, TT, C_NE, false>(a, b, (TT)k, mask);                     \
    case 64 + TCODE * 8 + C_LT: return pred4<NT, G, TT, C_LT, true>(a, b, (TT)0, mask);                 \
    case 64 + TCODE * 8 + C_LE: return pred4<NT, G, TT, C_LE, true>(a, b, (TT)0, mask);                 \
    case 64 + TCODE * 8 + C_GT: return pred4<NT, G, TT, C_GT, true>(a, b, (TT)0, mask);                 \
    case 64 + TCODE * 8 + C_GE: return pred4<NT, G, TT, C_GE, true>(a, b, (TT)0, mask);                 \
    case 64 + TCODE * 8 + C_EQ: return pred4<NT, G, TT, C_EQ, true>(a, b, (TT)0, mask);                 \
    case 64 + TCODE * 8 + C_NE: return pred4<NT, G, TT, C_NE, true>(a, b, (TT)0, mask);

template <int NT, int G>
__device__ __noinline__ uint32_t run_pred4(uint32_t code, int64_t k, const char *a, const char *b, uint32_t mask)
{
    switch (code) {
        RW_PRED4_CASES(int32_t, T_I32)
        RW_PRED4_CASES(uint32_t, T_U32)
        RW_PRED4_CASES(int64_t, T_I64)
        RW_PRED4_CASES(uint64_t, T_U64)
        RW_PRED4_CASES(uint8_t, T_U8)
    }
    return mask;
}

// dst = a OP (b | k) over the thread's rows; operands of another type are converted
// into T (mod 2^w), as in chain.cuh expr_loop
template <int NT, int G, typename T, int OP, bool BSLOT>
__device__ __forceinline__ void expr4(char *dst, const char *a, int ta, const char *b, int tb, T k)
{
    constexpr int TT = sizeof(T) == 8 ? (std::is_signed<T>::value ? T_I64 : T_U64)
                                      : (std::is_signed<T>::value ? T_I32 : T_U32);
    const bool sa = (ta == TT) || (sizeof(T) == 4 && (ta == T_I32 || ta == T_U32)) ||
                    (sizeof(T) == 8 && (ta == T_I64 || ta == T_U64));
    const bool sb = (tb == TT) || (sizeof(T) == 4 && (tb == T_I32 || tb == T_U32)) ||
                    (sizeof(T) == 8 && (tb == T_I64 || tb == T_U64));
#pragma unroll
    for (int g = 0; g < G; g++) {
        const int r0 = row4<NT>(g);
        V4<T> x, y, o;
        if (OP != E_CONST) {
            if (sa) x = ld4<T>(a, r0);
            else { const V4<uint64_t> e = ld4_ext(a, ta, r0); for (int q = 0; q < 4; q++) x.v[q] = (T)e.v[q]; }
        }
        if (BSLOT) {
            if (sb) y = ld4<T>(b, r0);
            else { const V4<uint64_t> e = ld4_ext(b, tb, r0); for (int q = 0; q < 4; q++) y.v[q] = (T)e.v[q]; }
        }
#pragma unroll
        for (int q = 0; q < 4; q++)
            o.v[q] = ev<T, OP>(OP == E_CONST ? (T)0 : x.v[q], BSLOT ? y.v[q] : k);
        st4<T>(dst, r0, o);
    }
}

template <int NT, int G, typename T>
__device__ __forceinline__ void mulaff4(char *dst, const char *a, const char *b, T k, bool neg)
{
    typedef typename std::make_unsigned<T>::type U;
#pragma unroll
    for (int g = 0; g < G; g++) {
        const int r0 = row4<NT>(g);
        const V4<T> x = ld4<T>(a, r0), y = ld4<T>(b, r0);
        V4<T> o;
#pragma unroll
        for (int q = 0; q < 4; q++)
            o.v[q] = (T)((U)x.v[q] * (neg ? (U)k - (U)y.v[q] : (U)k + (U)y.v[q]));
        st4<T>(dst, r0, o);
    }
}

#define RW_EXPR4_CASES(TT, TCODE)                                                                           \
    case TCODE * 8 + E_COPY: expr4<NT, G, TT, E_COPY, false>(dst, a, ta, b, tb, (TT)k); return;             \
    case TCODE * 8 + E_CONST: expr4<NT, G, TT, E_CONST, false>(dst, a, ta, b, tb, (TT)k); return;           \
    case TCODE * 8 + E_ADD: expr4<NT, G, TT, E_ADD, false>(dst, a, ta, b, tb, (TT)k); return;               \
    case TCODE * 8 + E_SUB: expr4<NT, G, TT, E_SUB, false>(dst, a, ta, b, tb, (TT)k); return;               \
    case TCODE * 8 + E_MUL: expr4<NT, G, TT, E_MUL, false>(dst, a, ta, b, tb, (TT)k); return;               \
    case TCODE * 8 + E_DIVC: expr4<NT, G, TT, E_DIVC, false>(dst, a, ta, b, tb, (TT)k); return;             \
    case TCODE * 8 + E_RSUB: expr4<NT, G, TT, E_RSUB, false>(dst, a, ta, b, tb, (TT)k); return;             \
    case 64 + TCODE * 8 + E_ADD: expr4<NT, G, TT, E_ADD, true>(dst, a, ta, b, tb, (TT)0); return;           \
    case 64 + TCODE * 8 + E_SUB: expr4<NT, G, TT, E_SUB, true>(dst, a, ta, b, tb, (TT)0); return;           \
    case 64 + TCODE * 8 + E_MUL: expr4<NT, G, TT, E_MUL, true>(dst, a, ta, b, tb, (TT)0); return;           \
    case 64 + TCODE * 8 + E_MULAFF: mulaff4<NT, G, TT>(dst, a, b, (TT)k, (tb & kNegB) != 0); return;

template <int NT, int G>
__device__ __noinline__ void run_expr4(uint32_t code, int ta, int tb, int64_t k, char *dst, const char *a, const char *b)
{
    switch (code) {
        RW_EXPR4_CASES(int32_t, T_I32)
        RW_EXPR4_CASES(uint32_t, T_U32)
        RW_EXPR4_CASES(int64_t, T_I64)
        RW_EXPR4_CASES(uint64_t, T_U64)
    }
}

// The fused program over the thread's rows (§4.3.1: SELECT / PROJECT in order,
// in the same thread, no synchronisation between thread-dependent operators)
template <int NT, int G>
__device__ __forceinline__ uint32_t run_ops4(const ChainProg &P, int op0, int op1, const char *stage, char *scratch,
                                             uint32_t mask)
{
#pragma unroll 1
    for (int i = op0; i < op1; i++) {
        const uint32_t kind = P.ops[i].kind, code = P.ops[i].code;
        const int64_t k = P.ops[i].k;
        const char *a = loc_ptr(P.ops[i].a, stage, scratch);
        const char *b = loc_ptr(P.ops[i].b, stage, scratch);
        if (kind == K_PRED) {
            // inline fast paths for 32-bit column-vs-constant atoms
            if (code == T_I32 * 8 + C_LT)
                mask = pred4<NT, G, int32_t, C_LT, false>(a, b, (int32_t)k, mask);
            else if (code == T_U32 * 8 + C_LT)
                mask = pred4<NT, G, uint32_t, C_LT, false>(a, b, (uint32_t)k, mask);
            else
                mask = run_pred4<NT, G>(code, k, a, b, mask);
        } else {
            run_expr4<NT, G>(code, P.ops[i].ta, P.ops[i].tb, k, (char *)loc_ptr(P.ops[i].dst, stage, scratch), a, b);
        }
    }
    return mask;
}

// Compacted-store slow path of the emitting kernels: the survivors of the thread's
// groups (positions sp) of one column, into a circular ring whose segment for this
// column starts at byte `so` and wraps at R.
template <int NT, int G>
__device__ __forceinline__ void wrap_scatter(char *ring, uint32_t R, uint32_t so, int w, const char *src, uint32_t m,
                                          const uint32_t (&sp)[G][4])
{
    for (int g = 0; g < G; g++) {
        const uint32_t m4 = (m >> (4 * g)) & 15u;
        if (!m4)
            continue;
        const int r0 = row4<NT>(g);
        for (int q = 0; q < 4; q++) {
            if (!((m4 >> q) & 1u))
                continue;
            uint32_t b = so + sp[g][q] * (uint32_t)w;
            if (b >= R)
                b -= R;
            if (w == 4) *(uint32_t *)(ring + b) = ((const uint32_t *)src)[r0 + q];
            else if (w == 8) *(uint64_t *)(ring + b) = ((const uint64_t *)src)[r0 + q];
            else ring[b] = src[r0 + q];
        }
    }
}

}  // namespace rw
