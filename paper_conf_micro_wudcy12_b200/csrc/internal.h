// internal.h — structures shared by the plan builder (host C++) and the sm_100a
// kernels.  Not part of the public ABI (that is include/rw.h).
//
// A fused group is lowered to a ChainProg: a small register-free "micro-op"
// program over SLOTS.  A slot is one column of the current tile held in shared
// memory (input slots are filled by TMA bulk copies or by the join expansion;
// computed slots hold PROJECT/arithmetic results).  The paper passes
// thread-dependent intermediates in registers (§4.3.1); here the whole
// tile is resident in smem and the per-row `match` bit stays in a register,
// which keeps the program interpretable without code generation (DESIGN.md
// "What differs from the paper").
#pragma once
#include <stdint.h>

#if !defined(__CUDACC__) && !defined(__host__)
#define __host__
#define __device__
#endif

namespace rw {

constexpr int kMaxSlots = 24;
constexpr int kMaxOps = 48;
constexpr int kMaxOut = 32;
constexpr int kMaxGroupCols = 8;
constexpr int kMaxAggs = 16;
constexpr int kThreads = 256;        // threads per CTA for every chain kernel
constexpr int kScanItems = 8;        // rows per thread per tile in the scan kernel (T = 2048)
constexpr int kMaxAggSlots = 4096;
constexpr int kMaxBranch = 4;        // input-dependence fusion: SELECT/PROJECT chains sharing one scan
constexpr int kRegD = 6;             // register aggregate terminal: groups x sums held per thread
constexpr int kRegA = 5;             // sums held per thread per group
constexpr int kNarrowNT = 576;       // aggregate variant specialised for 5 sums with 2 narrow (TPC-H Q1 shape)
constexpr int kNarrowItems = 4;      // rows per thread of that variant (tile 2304)

enum Type : uint8_t { T_I32 = 0, T_U32 = 1, T_I64 = 2, T_U64 = 3, T_U8 = 4 };
enum Cmp : uint8_t { C_LT = 0, C_LE = 1, C_GT = 2, C_GE = 3, C_EQ = 4, C_NE = 5 };
enum OpKind : uint8_t { K_PRED = 0, K_EXPR = 1 };
enum ExprOp : uint8_t { E_COPY = 0, E_CONST = 1, E_ADD = 2, E_SUB = 3, E_MUL = 4, E_DIVC = 5, E_RSUB = 6,
                        E_MULAFF = 7 };   // dst = a * (k + b), or a * (k - b) when tb has kNegB set
constexpr uint8_t kNegB = 0x80;

__host__ __device__ inline int type_width(int t) { return t == T_U8 ? 1 : (t == T_I64 || t == T_U64) ? 8 : 4; }
__host__ __device__ inline bool type_signed(int t) { return t == T_I32 || t == T_I64; }

struct SlotDesc {
    uint8_t type;
    uint8_t is_input;   // 1: lives in the (multi-buffered) stage; 0: lives in scratch
    uint16_t pad;
    uint32_t off;       // byte offset of the slot column inside stage / scratch
};

// A smem location of a slot column, resolved on the host: bit 31 set = in the
// scratch tile (computed columns), else in the input stage; low bits = byte offset.
constexpr uint32_t kLocScratch = 0x80000000u;

struct DevOp {
    uint8_t kind;       // K_PRED / K_EXPR
    uint8_t code;       // PRED: type*8 + cmp (+64: rhs is a slot); EXPR: type*8 + ExprOp (+64: b is a slot)
    uint8_t ta, tb;     // EXPR operand slot types (converted into the result type)
    uint32_t a, b, dst; // encoded locations (kLocScratch | offset)
    int64_t k;          // constant (rhs / operand b / divisor), already wrapped to the op type
};

struct ChainProg {
    int32_t nslots;
    int32_t nin;                        // slots [0, nin) are input slots
    int32_t nops;
    int32_t nout;
    SlotDesc slot[kMaxSlots];
    const void *in_ptr[kMaxSlots];      // scan kernel: global column base of each input slot
    DevOp ops[kMaxOps];
    int16_t out_slot[kMaxOut];
    uint32_t out_loc[kMaxOut];          // encoded smem location of each output column
    uint8_t out_w[kMaxOut];             // byte width of each output column
    void *out_ptr[kMaxOut];
    int64_t out_capacity;
    // aggregate terminal (is_agg): group code g = sum code_c * stride_c
    int32_t is_agg;
    int32_t ngc;
    int16_t gslot[kMaxGroupCols];
    uint32_t g_loc[kMaxGroupCols];
    uint8_t g_type[kMaxGroupCols];
    int32_t gdomain[kMaxGroupCols];
    int32_t D;                          // product of domains
    int32_t nagg;                       // number of SUM accumulators (count is implicit, index 0)
    int16_t agg_slot[kMaxAggs];
    uint32_t agg_loc[kMaxAggs];
    uint8_t agg_type[kMaxAggs];
    uint8_t agg_unsigned[kMaxAggs];     // 1: u64 sum (unsigned partials)
    int64_t flush_rows;                 // rows a thread may add before its int64 partials can overflow
    int32_t agg_mode;                   // 0: thread-private partials in smem; 2: register one-hot (D <= kRegD, nagg <= kRegA)
    int32_t agg_narrow;                 // mode 2: the first agg_narrow sums are non-negative with |v| < 2^16 and
                                        // accumulate in 32-bit registers (flush_rows keeps them below 2^32)
    int32_t q1fused;                    // kNarrowNT instance: the Q1 program shape runs fused per row (agg_tile_q1)
    int32_t narrow_bits;                // every narrow value is < 2^narrow_bits (declared bounds); the kernel ORs
                                        // the narrow values of a tile and counts a violation into err[2]
    // input-dependence fusion (§4.4, Fig. 14(d)): nbranch chains over the same
    // staged tile, each with its own mask and compacted output.  Branch b runs ops
    // [br_op_end[b-1], br_op_end[b]) and writes output columns [br_out_end[b-1], br_out_end[b]).
    int32_t nbranch;                    // >= 1
    uint8_t br_op_end[kMaxBranch];
    uint8_t br_out_end[kMaxBranch];
    int64_t br_cap[kMaxBranch];         // output capacity of branch b (b = 0: out_capacity)
    uint8_t br_nw[kMaxBranch][3];       // output columns of branch b that are 1, 4 and 8 bytes wide
    uint32_t stage_bytes;               // bytes of one stage (all input slots, aligned)
    uint32_t scratch_bytes;             // bytes of scratch (computed slots)
};

// Launch-time scalars for the scan / join-expand kernels.
struct TileLaunch {
    int64_t n;                 // rows (scan) or join outputs (expand), if n_ptr == nullptr
    const int64_t *n_ptr;      // device row count written by an earlier kernel (else nullptr)
    int32_t stages;
    uint32_t out_bytes;        // scan kernel: bytes of the compacted-tile ring (per CTA)
    char *gring;               // scan kernel: global ring, gridDim.x * out_bytes bytes (nullptr: in smem)
    int32_t direct;            // scan kernel: no SELECT in the group, rows stored at their offsets
    int32_t use_tma;           // input slots may be bulk-copied (16B-aligned bases)
    uint32_t epoch;            // look-back epoch tag (1..65535)
    uint64_t *status;          // look-back status words, >= ntiles (per branch: + b * status_stride)
    int64_t status_stride;
    int64_t *br_n_dev[kMaxBranch];   // output row count of branch b >= 1 (branch 0: n_dev)
    uint32_t *ctrs;            // [0] tile counter, [1] done counter (reset by the last CTA)
    int64_t *n_dev;            // output row count
    unsigned long long *agg_acc;   // global 128-bit accumulators: D * (nagg+1) * 2 u64
    int32_t *err;              // [0] domain errors
    int32_t dbg;               // diagnostics: 1 = skip look-back (offset = tile * T, uncompacted),
                               // 2 = stream tiles only, 4 = per-tile phase timestamps into dbg_ts
    int32_t delay;             // emitting scan kernel: compute warps hold at most `delay` evaluated tiles
                               // (in their input stages) waiting for their global offsets
    uint32_t gring_bytes;      // emitting scan kernel: bytes of each CTA's L2 ring slice (gring != nullptr)
    uint64_t *dbg_ts;          // 12 globaltimer stamps per tile (claim, data, evaluated, offset, stored, writer start, ops, ballots, scattered, reserve start; join: records cached, gathered)
};

}  // namespace rw
