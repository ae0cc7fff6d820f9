// rw_api.cpp — C ABI (include/rw.h), plan builder, fusion legality / grouping
// (Algorithm 1 and 2 analogues, §4.1-4.2), lowering of each fused
// group to a ChainProg, and the stream-ordered executor.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <functional>
#include <map>
#include <sstream>
#include <string>
#include <vector>

#include "dist_kernels.h"
#include "kernels.h"
#include "plan.h"

using namespace rw;

namespace {

thread_local std::string g_err;

struct RwError {
    rw_status s;
    std::string msg;
};

[[noreturn]] void raise(rw_status s, const std::string &m) { throw RwError{s, m}; }

void cuda_check(cudaError_t e, const char *what)
{
    if (e != cudaSuccess)
        raise(RW_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

const i128 I128_BIG = ((i128)1) << 120;

i128 clampi(i128 v) { return v > I128_BIG ? I128_BIG : (v < -I128_BIG ? -I128_BIG : v); }

}  // namespace

namespace rw {

const char *dep_name(int d) { return d == DEP_THREAD ? "thread" : d == DEP_CTA ? "CTA" : "kernel"; }

Interval type_range(int t)
{
    switch (t) {
    case T_I32: return {INT32_MIN, INT32_MAX};
    case T_U32: return {0, UINT32_MAX};
    case T_I64: return {INT64_MIN, INT64_MAX};
    case T_U64: return {0, (i128)UINT64_MAX};
    default: return {0, 255};
    }
}

bool fits(const Interval &v, int t)
{
    Interval r = type_range(t);
    return v.lo >= r.lo && v.hi <= r.hi;
}

i128 wrap_to(int t, i128 v)
{
    unsigned __int128 u = (unsigned __int128)v;
    switch (t) {
    case T_I32: return (int32_t)(uint32_t)u;
    case T_U32: return (uint32_t)u;
    case T_I64: return (int64_t)(uint64_t)u;
    case T_U64: return (uint64_t)u;
    default: return (uint8_t)u;
    }
}

}  // namespace rw

// ===========================================================================
// Plan object
// ===========================================================================
struct Rel {
    std::vector<int> types;
    std::vector<const void *> cols;
    int64_t n_host = -1;          // known row count, or -1
    const int64_t *n_dev = nullptr;
    int64_t cap = 0;              // upper bound on rows
};

struct Lowered {
    ChainProg P;
    std::vector<int> in_src;      // input slot i <- source column in_src[i]
    int items = 8, stages = 2, ctas = 1;
    int tile = 2048;              // rows per tile
    int nt = 256;                 // compute threads per CTA (emit kernel: per team)
    int teams = 1;                // emit kernel: teams of nt compute threads on alternate tiles
    uint32_t gring_bytes = 0;     // per-CTA global ring bytes (0: ring in smem)
    bool direct = false;          // no SELECT: outputs written at their row offsets
    int ring = 0;                 // scan kernel: output ring entries
    uint32_t out_bytes = 0;       // bytes of one output ring entry
    std::vector<uint32_t> out_off;
    size_t smem = 0;
    bool agg = false;
    bool emit = false;            // compacting chain on the emitting scan kernel (scan_emit.cu)
    int delay = 1;                // emit: evaluated tiles a compute warp may hold for their offsets
    uint32_t warp_buf = 0;        // emit: per-warp compaction buffer bytes
    AggFinal F;
};

struct rw_plan {
    rw_plan_opts o;
    cudaStream_t stream = nullptr;
    int sms = 148;
    std::vector<Node> nodes;
    std::vector<int> inputs;      // node id of each declared input, declaration order
    // persistent scratch
    uint64_t *status = nullptr;
    int64_t status_cap = 0;
    int64_t status_used = 0;      // join groups: words handed out of `status` in this group
    uint32_t *ctrs = nullptr;     // 2 counters
    int64_t *cnt = nullptr;       // per-group row counts (grown)
    int cnt_cap = 0;
    int64_t *jtot = nullptr;      // join totals: 2 int64 per join group
    int64_t *jtot_host = nullptr; // pinned mirror
    int32_t *err = nullptr;       // [0] running domain errors, [1] last finalised; [2] running
                                  // declared-bound violations of narrow sums, [3] last finalised
    char *gring = nullptr;        // global compacted-tile rings (per CTA slices)
    size_t gring_cap = 0;
    std::map<int, unsigned long long *> agg_acc;
    uint32_t epoch = 0;
    int64_t launches = 0;
    bool defer_finalize = false;  // host-streamed aggregate: chunks accumulate, the last one finalises
    // host streaming (execute_host): copy streams, events and double-buffered chunk
    // buffers, created on first use and kept for the plan's lifetime
    struct HostStream {
        bool init = false;
        cudaStream_t sh = nullptr, sd = nullptr;
        cudaEvent_t ev[4][2];
        char *buf = nullptr;
        size_t bytes = 0;
        int64_t *hcnt = nullptr;
    } hs;
    std::vector<void *> temps;    // freed (stream-ordered) at the end of every execute
};

namespace {

void *dev_alloc(rw_plan *p, size_t bytes)
{
    void *ptr = nullptr;
    if (bytes == 0)
        bytes = 16;
    cudaError_t e = cudaMallocAsync(&ptr, bytes, p->stream);
    if (e == cudaErrorMemoryAllocation)
        raise(RW_E_OOM, "cudaMallocAsync: out of device memory");
    cuda_check(e, "cudaMallocAsync");
    return ptr;
}

void *temp_alloc(rw_plan *p, size_t bytes)
{
    void *ptr = dev_alloc(p, bytes);
    p->temps.push_back(ptr);
    return ptr;
}

void free_temps(rw_plan *p)
{
    for (void *t : p->temps)
        cudaFreeAsync(t, p->stream);
    p->temps.clear();
}

void ensure_status(rw_plan *p, int64_t need)
{
    if (need <= p->status_cap)
        return;
    int64_t cap = std::max<int64_t>(need, 2 * p->status_cap);
    cap = std::max<int64_t>(cap, 4096);
    if (p->status)
        cudaFreeAsync(p->status, p->stream);
    p->status = (uint64_t *)dev_alloc(p, (size_t)cap * 8);
    cuda_check(cudaMemsetAsync(p->status, 0, (size_t)cap * 8, p->stream), "memset status");
    p->status_cap = cap;
}

uint32_t next_epoch(rw_plan *p)
{
    p->epoch++;
    if (p->epoch > 0xffff) {
        p->epoch = 1;
        if (p->status)
            cuda_check(cudaMemsetAsync(p->status, 0, (size_t)p->status_cap * 8, p->stream), "memset status");
    }
    return p->epoch;
}

const Node &node_at(const rw_plan *p, int id)
{
    if (id < 0 || id >= (int)p->nodes.size())
        raise(RW_E_ARG, "node id " + std::to_string(id) + " out of range");
    return p->nodes[id];
}

bool is_unary_chain(NodeKind k) { return k == N_SELECT || k == N_PROJECT; }

// ---------------------------------------------------------------------------
// Interval analysis of PROJECT expressions (reading A8; strict mode rejects wrap)
// ---------------------------------------------------------------------------
Interval expr_interval(const Node &in, const std::vector<rw_expr> &e, int i, std::vector<Interval> &memo,
                       std::vector<char> &done, bool strict)
{
    if (done[i])
        return memo[i];
    const rw_expr &x = e[i];
    Interval r;
    auto finish = [&](Interval v) {
        if (!fits(v, x.type)) {
            if (strict && (x.type == T_I64 || x.type == T_U64))
                raise(RW_E_OVERFLOW, "expression node " + std::to_string(i) + " may wrap in its 64-bit type");
            v = type_range(x.type);
        }
        return v;
    };
    switch (x.op) {
    case RW_COL: r = finish(in.bounds[x.a]); break;
    case RW_CONST: {
        i128 v = wrap_to(x.type, x.k);
        r = {v, v};
        break;
    }
    case RW_ADD: case RW_SUB: case RW_MUL: {
        Interval a = expr_interval(in, e, x.a, memo, done, strict);
        Interval b = expr_interval(in, e, x.b, memo, done, strict);
        // operands are first converted into x.type
        if (!fits(a, x.type)) a = type_range(x.type);
        if (!fits(b, x.type)) b = type_range(x.type);
        if (x.op == RW_ADD) r = {clampi(a.lo + b.lo), clampi(a.hi + b.hi)};
        else if (x.op == RW_SUB) r = {clampi(a.lo - b.hi), clampi(a.hi - b.lo)};
        else {
            auto m = [](i128 u, i128 v) {
                i128 au = u < 0 ? -u : u, av = v < 0 ? -v : v;
                if (au != 0 && av > I128_BIG / au)
                    return ((u < 0) != (v < 0)) ? -I128_BIG : I128_BIG;
                return u * v;
            };
            i128 c[4] = {m(a.lo, b.lo), m(a.lo, b.hi), m(a.hi, b.lo), m(a.hi, b.hi)};
            r = {*std::min_element(c, c + 4), *std::max_element(c, c + 4)};
        }
        r = finish(r);
        break;
    }
    case RW_DIVC: {
        Interval a = expr_interval(in, e, x.a, memo, done, strict);
        if (!fits(a, x.type)) a = type_range(x.type);
        i128 k = wrap_to(x.type, x.k);
        i128 c1 = a.lo / k, c2 = a.hi / k;
        r = {std::min(c1, c2), std::max(c1, c2)};
        if (a.lo <= 0 && a.hi >= 0) {
            r.lo = std::min<i128>(r.lo, 0);
            r.hi = std::max<i128>(r.hi, 0);
        }
        r = finish(r);
        break;
    }
    default: raise(RW_E_ARG, "bad expression op");
    }
    memo[i] = r;
    done[i] = 1;
    return r;
}

// ---------------------------------------------------------------------------
// Grouping: Algorithm 1 (drop kernel-dependence edges, connected components)
// and Algorithm 2 (greedy, earliest operator first, under the resource budget)
// analogues.  Each group becomes one kernel template instance.
// ---------------------------------------------------------------------------
struct Grouping {
    std::vector<Group> groups;
    std::vector<int> cuts;              // nodes split at by the resource budget (Algorithm 2)
    std::map<int, int> produced_by;     // node -> group index
    std::vector<int> consumers;         // within the reachable sub-DAG
    std::vector<char> reach;
    std::vector<std::string> notes;
};

void mark_reach(const rw_plan *p, int id, Grouping &G)
{
    if (G.reach[id])
        return;
    G.reach[id] = 1;
    const Node &n = p->nodes[id];
    if (n.in >= 0) mark_reach(p, n.in, G);
    if (n.left >= 0) mark_reach(p, n.left, G);
    if (n.right >= 0) mark_reach(p, n.right, G);
}

int make_group(const rw_plan *p, int id, Grouping &G);

int dep_group(const rw_plan *p, int id, Grouping &G)
{
    if (p->nodes[id].kind == N_INPUT)
        return -1;
    return make_group(p, id, G);
}

// SELECTs on the key column only, directly upstream of a JOIN input (single consumer):
// they keep or drop whole key runs, so the join's run matching applies them and the
// join reads their source relation (CTA dependence fused, Fig. 13; N2).
int absorb_key_selects(const rw_plan *p, int nd, const Grouping &G, Group &g, int &npred, int nkey)
{
    if (!p->o.fuse || nkey != 1)
        return nd;
    while (p->nodes[nd].kind == N_SELECT && G.consumers[nd] == 1) {
        const Node &sn = p->nodes[nd];
        bool keyonly = !sn.preds.empty();
        for (const rw_pred &a : sn.preds)
            keyonly = keyonly && a.col == 0 && !a.rhs_is_col;
        if (!keyonly || npred + (int)sn.preds.size() > kMaxKeyPreds)
            break;
        npred += (int)sn.preds.size();
        g.pre.push_back(nd);
        nd = sn.in;
    }
    return nd;
}

// A JOIN group (§4.3.2): key SELECTs on its inputs are absorbed into the
// run matching (N2), and a left input that is itself a single-consumer JOIN on the same
// key (CTA dependence, Fig. 8(b); pattern (b) of Fig. 14) is absorbed too: the
// group then joins three inputs in one expansion (mixed radix (i, j, k)).
void setup_join(const rw_plan *p, int jid, Grouping &G, Group &g)
{
    g.kind = G_JOIN;
    g.join = jid;
    const Node &j = p->nodes[jid];
    int np = 0;
    const int left = j.left;
    const Node &ln = p->nodes[left];
    // an input's upstream SELECT / PROJECT chain (single consumers): key SELECTs go to the
    // run matching; the rest becomes the side's pre-chain, evaluated on the gathered rows
    auto side_src = [&](int start, int side) {
        int nd = absorb_key_selects(p, start, G, g, np, j.nkey);
        while (p->o.fuse && p->o.reserved[6] != 7 && is_unary_chain(p->nodes[nd].kind) && G.consumers[nd] == 1 &&
               p->nodes[nd].nkey_sorted >= j.nkey) {
            g.prechain[side].insert(g.prechain[side].begin(), nd);
            nd = absorb_key_selects(p, p->nodes[nd].in, G, g, np, j.nkey);
        }
        return nd;
    };
    if (p->o.fuse && ln.kind == N_JOIN && G.consumers[left] == 1 && ln.nkey == j.nkey && p->o.reserved[6] != 5) {
        g.join_in = left;
        g.jl = side_src(ln.left, 0);
        g.jr = side_src(ln.right, 1);
        g.jc = side_src(j.right, 2);
    } else {
        g.jl = side_src(left, 0);
        g.jr = side_src(j.right, 1);
    }
    for (int src : {g.jl, g.jr, g.jc}) {
        if (src < 0) continue;
        const int d = dep_group(p, src, G);
        if (d >= 0) g.deps.push_back(d);
    }
}

int make_group(const rw_plan *p, int id, Grouping &G)
{
    auto it = G.produced_by.find(id);
    if (it != G.produced_by.end())
        return it->second;
    const bool fuse = p->o.fuse != 0;
    const Node &n = p->nodes[id];
    Group g;
    g.out = id;
    int cur = id;
    if (n.kind == N_AGG) {
        g.agg = id;
        cur = n.in;
        if (fuse && p->nodes[cur].kind == N_JOIN && G.consumers[cur] == 1) {
            // JOIN -> AGG: the aggregate is the join expansion's terminal (CTA dependence)
            setup_join(p, cur, G, g);
            G.groups.push_back(g);
            return G.produced_by[id] = (int)G.groups.size() - 1;
        }
        if (!fuse || !is_unary_chain(p->nodes[cur].kind) || G.consumers[cur] != 1) {
            // AGG directly over a relation (or operator-at-a-time mode)
            g.kind = G_SCAN;
            g.source = cur;
            int d = dep_group(p, cur, G);
            if (d >= 0) g.deps.push_back(d);
            G.groups.push_back(g);
            return G.produced_by[id] = (int)G.groups.size() - 1;
        }
    }
    if (n.kind == N_SETOP) {
        // set operators read both (materialised, fully sorted) inputs by merge path
        g.kind = G_SET;
        g.join = id;
        int a = dep_group(p, n.left, G), b = dep_group(p, n.right, G);
        if (a >= 0) g.deps.push_back(a);
        if (b >= 0) g.deps.push_back(b);
        G.groups.push_back(g);
        return G.produced_by[id] = (int)G.groups.size() - 1;
    }
    if (n.kind == N_JOIN) {
        setup_join(p, id, G, g);
        G.groups.push_back(g);
        return G.produced_by[id] = (int)G.groups.size() - 1;
    }
    // cur is SELECT / PROJECT: absorb producers while the edge is thread dependence
    // with a single consumer (§4.3.1)
    std::vector<int> chain{cur};
    int src = p->nodes[cur].in;
    while (fuse && is_unary_chain(p->nodes[src].kind) && G.consumers[src] == 1) {
        chain.insert(chain.begin(), src);
        src = p->nodes[src].in;
    }
    if (!fuse) {
        // operator-at-a-time: one operator per group
        chain.assign(1, cur);
        src = p->nodes[cur].in;
    }
    // JOIN -> chain -> AGG: the join expansion's aggregate terminal (X -> AGG is CTA
    // dependence: block reduction + one global atomic stage), handled below with the
    // other JOIN -> SELECT / PROJECT groups
    g.chain = chain;
    if (fuse && p->nodes[src].kind == N_JOIN && G.consumers[src] == 1) {
        // JOIN -> SELECT/PROJECT: fused into the join expansion (CTA dependence)
        setup_join(p, src, G, g);
    } else {
        g.kind = G_SCAN;
        g.source = src;
        int d = dep_group(p, src, G);
        if (d >= 0) g.deps.push_back(d);
    }
    G.groups.push_back(g);
    return G.produced_by[id] = (int)G.groups.size() - 1;
}

// raw column types of a join group's inputs, side by side (its input slot space)
std::vector<int> join_src_types(const rw_plan *p, const Group &g)
{
    std::vector<int> t;
    for (int src : {g.jl, g.jr, g.jc})
        if (src >= 0)
            for (int ty : p->nodes[src].types) t.push_back(ty);
    return t;
}

Grouping build_groups_once(const rw_plan *p, int out_node, const std::vector<int> &cuts)
{
    Grouping G;
    G.consumers.assign(p->nodes.size(), 0);
    G.reach.assign(p->nodes.size(), 0);
    mark_reach(p, out_node, G);
    // nodes Algorithm 2 split at (resource budget): their output is materialised, so
    // they count as having a further consumer
    for (int c : cuts)
        G.consumers[c] += 1;
    G.cuts = cuts;
    for (size_t i = 0; i < p->nodes.size(); i++) {
        if (!G.reach[i]) continue;
        const Node &n = p->nodes[i];
        if (n.in >= 0) G.consumers[n.in]++;
        if (n.left >= 0) G.consumers[n.left]++;
        if (n.right >= 0) G.consumers[n.right]++;
    }
    G.consumers[out_node]++;   // the caller consumes the output
    make_group(p, out_node, G);
    return G;
}

// Dependence class of edge producer -> consumer (legality rules SURVEY §8(a)).
int classify_edge(const rw_plan *p, int prod, int cons)
{
    const Node &a = p->nodes[prod];
    const Node &b = p->nodes[cons];
    if (a.kind == N_AGG)
        return DEP_KERNEL;                       // AGG behaves like a global barrier
    if (b.kind == N_SELECT || b.kind == N_PROJECT)
        return DEP_THREAD;                       // Fig. 8(a)
    if (b.kind == N_JOIN)
        return a.nkey_sorted >= b.nkey ? DEP_CTA : DEP_KERNEL;   // Fig. 8(b); unsorted -> SORT boundary
    if (b.kind == N_AGG)
        return DEP_CTA;                          // block reduction + one global atomic stage
    if (b.kind == N_SETOP)
        return a.nkey_sorted >= (int)a.types.size() ? DEP_CTA : DEP_KERNEL;   // merge path over whole tuples
    return DEP_KERNEL;
}

// ---------------------------------------------------------------------------
// Lowering of one group to a ChainProg
// ---------------------------------------------------------------------------
// host form of a micro-op (slot ids); encoded into DevOp locations after layout
struct HOp {
    uint8_t kind, op, type, b_is_slot;
    int16_t dst, a, b, pad;
    int64_t k;
    int br;                     // branch (input-dependence fusion), ops are in branch order
};

struct SlotB {
    int type;
    bool input;
    int src;
    int last_use;
    int region;
};

constexpr int kInf = 1 << 30;
constexpr size_t kSmemLimit = 227 * 1024;

size_t al128(size_t x) { return (x + 127) / 128 * 128; }

void lower(rw_plan *p, const Group &g, const std::vector<int> &src_types, Lowered &L)
{
    std::memset(&L.P, 0, sizeof(L.P));
    std::memset(&L.F, 0, sizeof(L.F));
    std::vector<SlotB> slots;
    std::vector<HOp> ops;
    std::vector<int> src_slot(src_types.size(), -1);
    auto get_src = [&](int c) {
        if (src_slot[c] < 0) {
            slots.push_back({src_types[c], true, c, -1, -1});
            src_slot[c] = (int)slots.size() - 1;
        }
        return src_slot[c];
    };
    auto new_slot = [&](int type) {
        slots.push_back({type, false, -1, -1, -1});
        return (int)slots.size() - 1;
    };
    std::vector<int> cur(src_types.size());
    for (size_t c = 0; c < cur.size(); c++)
        cur[c] = -1 - (int)c;
    auto resolve = [&](int v) { return v >= 0 ? v : get_src(-1 - v); };
    int cur_br = 0;
    auto push = [&](const HOp &o) {
        if ((int)ops.size() >= kMaxOps)
            raise(RW_E_UNSUPPORTED, "fused group exceeds the micro-op budget");
        ops.push_back(o);
        ops.back().br = cur_br;
    };
    const int nbr = g.branches.empty() ? 1 : (int)g.branches.size();
    if (nbr > kMaxBranch)
        raise(RW_E_UNSUPPORTED, "more than 4 input-dependent branches in one group");
    if (nbr > 1 && g.agg >= 0)
        raise(RW_E_UNSUPPORTED, "input-dependence fusion of aggregates");
    std::vector<int> term;
    std::vector<int> term_end;        // per branch: end of its terminal columns in term
    for (cur_br = 0; cur_br < nbr; cur_br++) {
    const std::vector<int> &chain_b = g.branches.empty() ? g.chain : g.branches[cur_br];
    cur.resize(src_types.size());
    for (size_t c = 0; c < src_types.size(); c++)
        cur[c] = -1 - (int)c;
    // one SELECT / PROJECT node applied to the column references `cur` (slot ids, or
    // -1-c for source column c not yet loaded)
    auto apply = [&](int nid, std::vector<int> &cur) {
        const Node &nd = p->nodes[nid];
        if (nd.kind == N_SELECT) {
            for (const rw_pred &a : nd.preds) {
                HOp o{};
                o.kind = K_PRED;
                o.op = (uint8_t)a.op;
                o.a = (int16_t)resolve(cur[a.col]);
                o.type = (uint8_t)slots[o.a].type;
                o.dst = -1;
                if (a.rhs_is_col) {
                    o.b_is_slot = 1;
                    o.b = (int16_t)resolve(cur[a.rhs_col]);
                } else {
                    o.b = -1;
                    o.k = (int64_t)wrap_to(o.type, a.rhs_const);
                }
                push(o);
            }
        } else {   // PROJECT
            const std::vector<rw_expr> &e = nd.exprs;
            // value of an expression node: slot id (>= 0) or a constant
            std::vector<int> vslot(e.size(), -2);
            std::vector<i128> vconst(e.size(), 0);
            std::vector<char> isconst(e.size(), 0);
            std::function<void(int)> ev = [&](int i) {
                if (vslot[i] != -2 || isconst[i])
                    return;
                const rw_expr &x = e[i];
                if (x.op == RW_COL) {
                    int s = resolve(cur[x.a]);
                    if (slots[s].type == x.type) {
                        vslot[i] = s;
                    } else {
                        int d = new_slot(x.type);
                        HOp o{};
                        o.kind = K_EXPR; o.op = E_COPY; o.type = (uint8_t)x.type;
                        o.dst = (int16_t)d; o.a = (int16_t)s; o.b = -1;
                        push(o);
                        vslot[i] = d;
                    }
                    return;
                }
                if (x.op == RW_CONST) {
                    isconst[i] = 1;
                    vconst[i] = wrap_to(x.type, x.k);
                    return;
                }
                ev(x.a);
                if (x.op != RW_DIVC)
                    ev(x.b);
                const int t = x.type;
                auto fold = [&](i128 a, i128 b) -> i128 {
                    unsigned __int128 ua = (unsigned __int128)wrap_to(t, a), ub = (unsigned __int128)wrap_to(t, b);
                    switch (x.op) {
                    case RW_ADD: return wrap_to(t, (i128)(ua + ub));
                    case RW_SUB: return wrap_to(t, (i128)(ua - ub));
                    case RW_MUL: return wrap_to(t, (i128)(ua * ub));
                    default: {
                        i128 sa = wrap_to(t, a), sb = wrap_to(t, b);
                        return wrap_to(t, sa / sb);
                    }
                    }
                };
                if (x.op == RW_DIVC) {
                    if (isconst[x.a]) {
                        isconst[i] = 1;
                        vconst[i] = fold(vconst[x.a], x.k);
                        return;
                    }
                    int d = new_slot(t);
                    HOp o{};
                    o.kind = K_EXPR; o.op = E_DIVC; o.type = (uint8_t)t;
                    o.dst = (int16_t)d; o.a = (int16_t)vslot[x.a]; o.b = -1;
                    o.k = (int64_t)wrap_to(t, x.k);
                    push(o);
                    vslot[i] = d;
                    return;
                }
                if (isconst[x.a] && isconst[x.b]) {
                    isconst[i] = 1;
                    vconst[i] = fold(vconst[x.a], vconst[x.b]);
                    return;
                }
                int d = new_slot(t);
                HOp o{};
                o.kind = K_EXPR; o.type = (uint8_t)t; o.dst = (int16_t)d; o.b = -1;
                const uint8_t base = x.op == RW_ADD ? E_ADD : x.op == RW_SUB ? E_SUB : E_MUL;
                if (isconst[x.b]) {
                    o.op = base; o.a = (int16_t)vslot[x.a]; o.k = (int64_t)wrap_to(t, vconst[x.b]);
                } else if (isconst[x.a]) {
                    o.op = base == E_SUB ? E_RSUB : base;
                    o.a = (int16_t)vslot[x.b]; o.k = (int64_t)wrap_to(t, vconst[x.a]);
                } else {
                    o.op = base; o.a = (int16_t)vslot[x.a]; o.b = (int16_t)vslot[x.b]; o.b_is_slot = 1;
                }
                push(o);
                vslot[i] = d;
            };
            std::vector<int> next;
            for (int r : nd.roots) {
                ev(r);
                if (isconst[r]) {
                    int d = new_slot(e[r].type);
                    HOp o{};
                    o.kind = K_EXPR; o.op = E_CONST; o.type = (uint8_t)e[r].type;
                    o.dst = (int16_t)d; o.a = -1; o.b = -1; o.k = (int64_t)vconst[r];
                    push(o);
                    next.push_back(d);
                } else {
                    next.push_back(vslot[r]);
                }
            }
            cur = next;
        }
        };
    if (g.kind == G_JOIN) {
        // join group: the input slots are the raw columns of the join inputs side by side
        // (A, B[, C]); each side's pre-chain (SELECT / key-preserving PROJECT fused
        // upstream of the JOIN, Fig. 13) runs on its own columns: a predicate of
        // a side holds for a candidate iff it holds for that side's row (bag semantics,
        // order kept), so it is evaluated on the gathered candidate.  Then the join output
        // (key, A rest, B rest[, C rest]) is assembled and the downstream chain follows.
        const int nk = p->nodes[g.join].nkey;
        const int sides = g.join_in >= 0 ? 3 : 2;
        const int srcn[3] = {g.jl, g.jr, g.jc};
        std::vector<int> out;
        int base = 0;
        for (int sd = 0; sd < sides; sd++) {
            const int nc = (int)p->nodes[srcn[sd]].types.size();
            std::vector<int> cs(nc);
            for (int c = 0; c < nc; c++)
                cs[c] = -1 - (base + c);
            for (int nid : g.prechain[sd])
                apply(nid, cs);
            for (size_t c = sd == 0 ? 0 : nk; c < cs.size(); c++)
                out.push_back(cs[c]);
            base += nc;
        }
        cur = out;
    }
    for (int nid : chain_b)
        apply(nid, cur);
    if (nbr > 1) {
        for (int v : cur)
            term.push_back(resolve(v));
        term_end.push_back((int)term.size());
    }
    }   // branches

    // terminal
    int narrow_n = 0;
    bool narrow_all64 = true;
    unsigned __int128 narrow_flush = 0;
    if (nbr > 1) {
        // materialising terminals collected per branch above
    } else if (g.agg >= 0) {
        const Node &a = p->nodes[g.agg];
        L.agg = true;
        L.P.is_agg = 1;
        L.P.ngc = (int)a.gcols.size();
        L.P.D = a.D;
        for (size_t c = 0; c < a.gcols.size(); c++) {
            int s = resolve(cur[a.gcols[c]]);
            L.P.gslot[c] = (int16_t)s;
            L.P.gdomain[c] = a.gdomain[c];
            term.push_back(s);
        }
        int ns = 0;
        const Node &an = p->nodes[a.in];
        // flush period: rows whose |values| sum cannot leave int64 (uint64 for u64 sums)
        unsigned __int128 flush = ((unsigned __int128)1) << 40;
        L.F.nreq = (int)a.aggs.size();
        // sums whose values are non-negative and below 2^16 ("narrow") are numbered
        // first: the register terminal accumulates them in 32-bit registers
        std::vector<size_t> order_q;
        for (int pass = 0; pass < 2; pass++)
            for (size_t q = 0; q < a.aggs.size(); q++) {
                if (a.aggs[q].op != RW_SUM) continue;
                const Interval b = an.bounds[a.aggs[q].col];
                const bool nar = b.lo >= 0 && b.hi < 65536;
                if (nar == (pass == 0)) order_q.push_back(q);
            }
        narrow_n = 0;
        narrow_flush = ((unsigned __int128)1) << 40;
        int narrow_bits = 1;
        for (size_t q = 0; q < a.aggs.size(); q++)
            if (a.aggs[q].op != RW_SUM) {
                L.F.req_is_sum[q] = 0;
                L.F.req_acc[q] = 0;
            }
        for (size_t q : order_q) {
                int s = resolve(cur[a.aggs[q].col]);
                L.P.agg_slot[ns] = (int16_t)s;
                const bool uns = slots[s].type == T_U64;
                L.P.agg_unsigned[ns] = uns;
                term.push_back(s);
                Interval b = an.bounds[a.aggs[q].col];
                unsigned __int128 mx = (unsigned __int128)(b.hi < 0 ? -b.hi : b.hi);
                unsigned __int128 mn = (unsigned __int128)(b.lo < 0 ? -b.lo : b.lo);
                if (mn > mx) mx = mn;
                if (mx == 0) mx = 1;
                unsigned __int128 lim = uns ? (unsigned __int128)UINT64_MAX : (unsigned __int128)INT64_MAX;
                flush = std::min(flush, std::max<unsigned __int128>(1, lim / mx));
                narrow_all64 = narrow_all64 && (slots[s].type == T_I64 || slots[s].type == T_U64);
                if (b.lo >= 0 && b.hi < 65536) {
                    // the device checks every narrow value against 2^narrow_bits (an OR per
                    // row), so the flush period is taken from that power of two
                    int bits = 1;
                    while (((i128)1 << bits) <= b.hi) bits++;
                    narrow_bits = std::max(narrow_bits, bits);
                    narrow_n++;
                    narrow_flush = std::min(narrow_flush, (unsigned __int128)UINT32_MAX / (((unsigned __int128)1 << narrow_bits) - 1));
                }
                L.F.req_is_sum[q] = 1;
                L.F.req_acc[q] = (int16_t)(1 + ns);
                ns++;
        }
        L.P.nagg = ns;
        L.P.narrow_bits = narrow_bits;
        L.P.flush_rows = (int64_t)flush;
        L.F.D = a.D;
        L.F.NA = ns + 1;
        L.F.ngc = L.P.ngc;
        for (int c = 0; c < L.P.ngc; c++) {
            L.F.gdomain[c] = a.gdomain[c];
            L.F.gtype[c] = (uint8_t)p->nodes[g.out].types[c];
        }
    } else {
        for (int v : cur)
            term.push_back(resolve(v));
    }
    if ((int)slots.size() > kMaxSlots)
        raise(RW_E_UNSUPPORTED, "fused group needs more than 24 tile columns");

    // peephole: MUL(x, y) with y = k + z or k - z (z a slot, k a constant, same type,
    // y used by nothing else) becomes one fused factor op dst = x * (k +- z)
    {
        std::vector<int> uses(slots.size(), 0), producer(slots.size(), -1);
        for (size_t i = 0; i < ops.size(); i++) {
            const HOp &o = ops[i];
            if (o.a >= 0) uses[o.a]++;
            if (o.b_is_slot && o.b >= 0) uses[o.b]++;
            if (o.kind == K_EXPR && o.dst >= 0) producer[o.dst] = (int)i;
        }
        for (int s : term) uses[s] += 2;
        std::vector<char> dead(ops.size(), 0);
        for (size_t i = 0; i < ops.size(); i++) {
            HOp &o = ops[i];
            if (o.kind != K_EXPR || o.op != E_MUL || !o.b_is_slot || o.a < 0 || o.b < 0) continue;
            for (int side = 0; side < 2; side++) {
                const int y = side ? o.a : o.b, x = side ? o.b : o.a;
                const int j = producer[y];
                if (j < 0 || dead[j] || uses[y] != 1) continue;
                const HOp &f = ops[j];
                if (f.kind != K_EXPR || f.b_is_slot || f.a < 0 || (f.op != E_ADD && f.op != E_RSUB)) continue;
                if (f.type != o.type || slots[f.a].type != o.type || slots[x].type != o.type) continue;
                if (slots[f.a].input == false && producer[f.a] > (int)i) continue;
                HOp m = o;
                m.op = E_MULAFF;
                m.a = (int16_t)x;
                m.b = (int16_t)f.a;
                m.b_is_slot = 1;
                m.k = f.k;
                m.pad = f.op == E_RSUB ? 1 : 0;          // 1: k - z
                o = m;
                dead[j] = 1;
                break;
            }
        }
        std::vector<HOp> kept;
        for (size_t i = 0; i < ops.size(); i++)
            if (!dead[i]) kept.push_back(ops[i]);
        ops.swap(kept);
    }

    // liveness
    for (size_t i = 0; i < ops.size(); i++) {
        const HOp &o = ops[i];
        if (o.a >= 0) slots[o.a].last_use = std::max(slots[o.a].last_use, (int)i);
        if (o.b_is_slot && o.b >= 0) slots[o.b].last_use = std::max(slots[o.b].last_use, (int)i);
    }
    for (int s : term)
        slots[s].last_use = kInf;

    // renumber: input slots first
    std::vector<int> order, remap(slots.size());
    for (size_t s = 0; s < slots.size(); s++)
        if (slots[s].input) order.push_back((int)s);
    const int nin = (int)order.size();
    for (size_t s = 0; s < slots.size(); s++)
        if (!slots[s].input) order.push_back((int)s);
    for (size_t i = 0; i < order.size(); i++)
        remap[order[i]] = (int)i;

    // scratch regions for computed slots (reuse freed regions of equal width)
    struct Region { int width; int owner; };
    std::vector<Region> regions;
    std::vector<int> dst_of_op(ops.size(), -1);
    for (size_t i = 0; i < ops.size(); i++) {
        if (ops[i].kind != K_EXPR) continue;
        for (Region &r : regions)
            if (r.owner >= 0 && slots[r.owner].last_use <= (int)i)
                r.owner = -1;
        const int d = ops[i].dst;
        const int w = type_width(slots[d].type);
        int got = -1;
        for (size_t r = 0; r < regions.size(); r++)
            if (regions[r].owner < 0 && regions[r].width == w) { got = (int)r; break; }
        if (got < 0) {
            regions.push_back({w, d});
            got = (int)regions.size() - 1;
        }
        regions[got].owner = d;
        slots[d].region = got;
    }

    // write ChainProg
    ChainProg &P = L.P;
    P.nslots = (int)slots.size();
    P.nin = nin;
    P.nops = (int)ops.size();
    P.nbranch = nbr;
    for (int b = 0; b < nbr; b++) {
        int e = 0;
        for (size_t i = 0; i < ops.size(); i++)
            if (ops[i].br <= b) e = (int)i + 1;
        P.br_op_end[b] = (uint8_t)e;
        P.br_out_end[b] = (uint8_t)(nbr > 1 ? term_end[b] : (int)term.size());
    }
    for (size_t i = 0; i < order.size(); i++) {
        const SlotB &sb = slots[order[i]];
        P.slot[i].type = (uint8_t)sb.type;
        P.slot[i].is_input = sb.input ? 1 : 0;
    }
    L.in_src.clear();
    for (int i = 0; i < nin; i++)
        L.in_src.push_back(slots[order[i]].src);
    std::vector<HOp> rops(ops);
    for (HOp &o : rops) {
        if (o.a >= 0) o.a = (int16_t)remap[o.a];
        if (o.b_is_slot && o.b >= 0) o.b = (int16_t)remap[o.b];
        if (o.dst >= 0) o.dst = (int16_t)remap[o.dst];
    }
    if (L.agg) {
        for (int c = 0; c < P.ngc; c++) P.gslot[c] = (int16_t)remap[P.gslot[c]];
        for (int q = 0; q < P.nagg; q++) P.agg_slot[q] = (int16_t)remap[P.agg_slot[q]];
    } else {
        if ((int)term.size() > kMaxOut)
            raise(RW_E_UNSUPPORTED, "more than 32 output columns");
        P.nout = (int)term.size();
        for (size_t j = 0; j < term.size(); j++)
            P.out_slot[j] = (int16_t)remap[term[j]];
    }

    // tile geometry, stages and CTAs per SM (resource budget, §4.3.3)
    auto layout = [&](int T) {
        uint32_t off = 0;
        for (int i = 0; i < nin; i++) {
            P.slot[i].off = off;
            off += (uint32_t)al128((size_t)T * type_width(P.slot[i].type));
        }
        P.stage_bytes = off;
        std::vector<uint32_t> roff(regions.size());
        uint32_t so = 0;
        for (size_t r = 0; r < regions.size(); r++) {
            roff[r] = so;
            so += (uint32_t)al128((size_t)T * regions[r].width);
        }
        P.scratch_bytes = so;
        for (size_t i = nin; i < order.size(); i++) {
            const SlotB &sb = slots[order[i]];
            P.slot[i].off = sb.region >= 0 ? roff[sb.region] : 0;
        }
        // resolve every slot reference to an encoded smem location
        auto loc = [&](int sl) -> uint32_t {
            if (sl < 0) return 0;
            return (P.slot[sl].is_input ? 0u : kLocScratch) | P.slot[sl].off;
        };
        for (size_t i = 0; i < rops.size(); i++) {
            const HOp &h = rops[i];
            DevOp d{};
            d.kind = h.kind;
            d.code = (uint8_t)(h.type * 8 + h.op + (h.b_is_slot ? 64 : 0));
            d.ta = h.a >= 0 ? P.slot[h.a].type : (uint8_t)h.type;
            d.tb = (h.b_is_slot && h.b >= 0) ? P.slot[h.b].type : (uint8_t)h.type;
            if (h.op == E_MULAFF && h.kind == K_EXPR && h.pad)
                d.tb |= kNegB;
            d.a = loc(h.a);
            d.b = h.b_is_slot ? loc(h.b) : 0;
            d.dst = h.dst >= 0 ? loc(h.dst) : 0;
            d.k = h.k;
            P.ops[i] = d;
        }
        for (int c = 0; c < P.nout; c++) {
            P.out_loc[c] = loc(P.out_slot[c]);
            P.out_w[c] = (uint8_t)type_width(P.slot[P.out_slot[c]].type);
        }
        for (int c = 0; c < P.ngc; c++) {
            P.g_loc[c] = loc(P.gslot[c]);
            P.g_type[c] = P.slot[P.gslot[c]].type;
        }
        for (int q = 0; q < P.nagg; q++) {
            P.agg_loc[q] = loc(P.agg_slot[q]);
            P.agg_type[q] = P.slot[P.agg_slot[q]].type;
        }
    };
    // aggregate terminal: warp reduce-by-key (agg_mode 1, per-warp 128-bit accumulators)
    // when the sums fit its unrolled loop and the per-warp accumulators are small;
    // else thread-private int64 partials (opts.reserved[7] == 1 forces the latter)
    // aggregate terminal: 2 = register one-hot (small D x sums, long flush period);
    // 0 = thread-private int64 partials in smem; 3 = per-row 128-bit global atomics
    // (group-bys whose partials exceed shared memory).  opts.reserved[7] == 1 forces 0.
    auto agg_mode_for = [&](int nt) -> int {
        if (!L.agg) return 0;
        const size_t slots = (size_t)P.D * (P.nagg + 1);
        if (p->o.reserved[7] == 1) return 0;
        if (P.D <= kRegD && P.nagg <= kRegA && P.flush_rows >= (1 << 16)) return 2;
        return slots * nt * 8 <= 150 * 1024 ? 0 : 3;
    };
    auto agg_bytes_for = [&](int nt) -> size_t {
        if (!L.agg) return 0;
        const size_t slots = (size_t)P.D * (P.nagg + 1);
        const size_t part = agg_mode_for(nt) == 0 ? slots * nt * 8 : 0;
        return part + al128(slots * 16);
    };
    if (L.agg && (size_t)P.D * (P.nagg + 1) > (size_t)kMaxAggSlots)
        raise(RW_E_UNSUPPORTED, "aggregate needs more than 4096 accumulators");

    if (g.kind == G_JOIN) {
        // join expansion (join2.cu k_join_emit): S stages of run records (TMA), two
        // gathered tiles (parity), scratch, and the compacted-output ring (resource
        // budget, §4.3.3)
        const int ways = g.join_in >= 0 ? 3 : 2;
        bool found = false;
        double best = -1;
        struct JV { int nt, items; };
        if (L.agg) {
            // register one-hot partials for small group-bys, else per-row global atomics;
            // the narrow 32-bit partials are a scan-kernel specialisation (not used here)
            P.agg_mode = (P.D <= kRegD && P.nagg <= kRegA && P.flush_rows >= (1 << 16)) ? 2 : 3;
            P.agg_narrow = 0;
        }
        for (JV jv : {JV{256, 8}, JV{512, 4}, JV{256, 4}}) {
            if (L.agg && !(jv.nt == 256 && jv.items == 8)) continue;
            const int items = jv.items, ntj = jv.nt;
            if (p->o.reserved[5] > 0 && items != p->o.reserved[5]) continue;
            if (p->o.reserved[4] == 7 ? ntj != 512 : (p->o.reserved[4] == 8 && ntj != 256)) continue;
            const int T = ntj * items;
            layout(T);
            size_t W = 0;
            for (int c = 0; c < P.nout; c++)
                W += (((size_t)T * type_width(P.slot[P.out_slot[c]].type)) + 15) / 16 * 16;
            if (L.agg)
                W = P.agg_mode == 2 ? al128((size_t)P.D * (P.nagg + 1) * 16) : 128;   // CTA accumulators, no ring
            const size_t RS = join_rec_stage_bytes(ways, T);
            const size_t base = join_emit_ctl_bytes() + 2 * (size_t)P.stage_bytes + (size_t)ways * T * 4 +
                                (size_t)T * 2 + P.scratch_bytes;
            for (int occ_t : {1, 2}) {
              if (p->o.ctas_per_sm > 0 ? occ_t != p->o.ctas_per_sm : occ_t != 1) continue;
              for (int S = 1; S <= 3; S++) {
                // one record stage is a candidate too: the next tile's records are then
                // fetched after the current tile releases its stage, but it lets the
                // 3-input group run 512 compute threads (measured C5 9.57 -> 8.21 ms)
                if (p->o.stages > 0 && S != p->o.stages) continue;
                const size_t per_cta = std::min(kSmemLimit, (size_t)(228 * 1024) / occ_t - 1024);
                if (base + S * RS + W > per_cta) continue;
                size_t Rb = (per_cta - base - S * RS) / 128 * 128;
                if (p->o.reserved[0] > 0) Rb = std::min(Rb, (size_t)p->o.reserved[0] * 1024);
                if (L.agg) Rb = W;
                if (Rb < W) continue;
                const size_t smem = base + S * RS + Rb;
                if (join_emit_occupancy(ntj, items, ways, smem, L.agg) < occ_t) continue;
                // measured (C3, C5): more compute warps first (512 x 4 beats 256 x 8 and,
                // for the 3-input group, 256 x 4 with the larger ring), then the tile, then
                // the ring's worst-case blocks
                const double q = (double)Rb / (double)W;
                const double sc = ntj * 1e6 + T * 1e2 + std::min(q, 4.0) * 10 + S;
                if (sc > best) {
                    best = sc;
                    L.items = items;
                    L.nt = ntj;
                    L.tile = T;
                    L.stages = S;
                    L.out_bytes = (uint32_t)Rb;
                    L.smem = smem;
                    L.ctas = occ_t;
                    found = true;
                }
              }
            }
        }
        if (!found)
            raise(RW_E_UNSUPPORTED, "join group exceeds the shared-memory budget");
        layout(L.tile);
        for (int c = 0; c < P.nout; c++) {
            const int w = type_width(P.slot[P.out_slot[c]].type);
            P.br_nw[0][w == 1 ? 0 : w == 4 ? 1 : 2]++;
        }
        return;
    }
    // Kernel choice for compacting chains: the emitting kernel (4-row vectors, shared +
    // L2 rings) when the chain filters at least twice (expected survival <= 1/4 under the
    // 50%-per-atom reading, small compacted tiles) or not at all (rows stored in place);
    // the L2-ring kernel below for single-atom filters (large compacted tiles) and for
    // input-dependence branches, where it measured faster.
    int npred_ops = 0;
    for (const HOp &h : ops)
        if (h.kind == K_PRED) npred_ops++;
    const bool use_emit = p->o.reserved[6] == 10 ||
                          (p->o.reserved[6] != 3 && nbr == 1 && (npred_ops == 0 || npred_ops >= 2));
    if (!L.agg && use_emit) {
        // Emitting scan kernel (scan_emit.cu): S input stages, each with its own scratch
        // for computed columns (a stage holds its tile until the tile's offset resolves),
        // per-thread hold words, and one compaction buffer per compute warp (resource
        // budget, §4.3.3).  Variants: compute threads x rows per thread.
        struct EVar { int nt, items, teams = 1; };
        std::vector<EVar> vars;
        if (p->o.reserved[4] == 3) vars.push_back({512, 8});
        else if (p->o.reserved[4] == 2) vars.push_back({256, 4});
        else if (p->o.reserved[4] == 4) vars.push_back({256, 8});
        else if (p->o.reserved[4] == 5) vars.push_back({256, 16});
        else if (p->o.reserved[4] == 6) vars.push_back({384, 8});
        else if (p->o.reserved[4] == 9) vars.push_back({384, 16});
        else if (p->o.reserved[4] == 7 && nbr == 1) vars.push_back({128, 16, 2});
        else if (p->o.reserved[4] == 8 && nbr == 1) vars.push_back({256, 8, 2});
        else if (nbr > 1) vars = {{256, 8}, {256, 4}};
        // 384 x 16: 12 compute warps on 6144-row tiles (measured C2 2.29 -> 2.06 ms: the
        // per-tile chain is latency-bound, so more warps and a larger tile both pay)
        else vars = {{384, 16}, {256, 16}, {256, 8}, {256, 4}};
        if (nbr > 1) {
            // the branch-loop (MULTI) instances exist for 256 x 8 and 256 x 4 (a 384 x 16
            // one measured slower on pattern (d): 5.24 vs 4.81 ms with the L2-ring kernel)
            std::vector<EVar> v2;
            for (const EVar &v : vars)
                if (v.teams == 1 && v.nt == 256 && (v.items == 8 || v.items == 4))
                    v2.push_back(v);
            vars = v2.empty() ? std::vector<EVar>{{256, 8}, {256, 4}} : v2;
        }
        const int want_stages_e = p->o.stages > 0 ? std::min(std::max(p->o.stages, 2), 8) : 0;
        bool direct_e = nbr == 1;
        for (const HOp &h : ops)
            if (h.kind == K_PRED) direct_e = false;
        double best = -1;
        const size_t want_ring_e = p->o.reserved[0] > 0 ? (size_t)p->o.reserved[0] * 1024 : 0;
        for (const EVar &v : vars) {
            const int T = v.nt * v.items;
            layout(T);
            const size_t SB = P.stage_bytes;
            size_t W = 0;                     // largest compacted block (every row survives)
            for (int b = 0; b < nbr && !direct_e; b++) {
                size_t wb = 0;
                for (int c = b ? P.br_out_end[b - 1] : 0; c < (int)P.br_out_end[b]; c++)
                    wb += ((size_t)T * type_width(P.slot[P.out_slot[c]].type) + 15) / 16 * 16;
                W = std::max(W, wb);
            }
            const size_t base = emit_ctl_bytes() + P.scratch_bytes;
            for (int occ_t : {1, 2}) {
                if (p->o.ctas_per_sm > 0 && occ_t != p->o.ctas_per_sm) continue;
                const size_t per_cta = std::min(kSmemLimit, (size_t)(228 * 1024) / occ_t - 1024);
                for (int S = 2; S <= 8; S++) {
                    if (want_stages_e && S != want_stages_e) continue;
                    if (base + (size_t)S * SB > per_cta) break;
                    // compacted-tile rings: shared memory (the remaining bytes) for blocks up to
                    // a quarter of it, and, when a worst-case block is larger than that, a
                    // per-CTA slice of an L2-resident buffer for the large blocks (>= 4 of them)
                    size_t Rs = direct_e ? 0 : (per_cta - base - (size_t)S * SB) / 128 * 128;
                    if (want_ring_e && !direct_e) Rs = std::min(Rs, want_ring_e);
                    if (p->o.reserved[6] == 9) Rs = 0;                   // diagnostics: L2 ring only
                    size_t Rg = 0;
                    if (!direct_e && W > Rs / 4 && p->o.reserved[6] != 8)
                        Rg = std::max<size_t>(4 * W, 128 * 1024) / 128 * 128;
                    if (!direct_e && !Rg && Rs < W) continue;
                    const size_t smem = base + (size_t)S * SB + Rs;
                    if (smem > per_cta) continue;
                    if (scan_emit_occupancy(v.nt, v.items, nbr > 1, smem, v.teams) < occ_t) continue;
                    // input bytes in flight per SM (capped: 128 KB covers the HBM latency;
                    // more stages only shrink the shared ring), the larger tile, then the
                    // larger shared ring
                    const double inflight = std::min<double>((double)occ_t * S * SB, 128.0 * 1024);
                    const double sc = inflight * 1e3 + (double)T * 64 * 1e3 + (double)std::min<size_t>(Rs, 96 * 1024) + S;
                    if (sc > best) {
                        best = sc;
                        L.items = v.items;
                        L.nt = v.nt;
                        L.teams = v.teams;
                        L.tile = T;
                        L.stages = S;
                        L.smem = smem;
                        L.ctas = occ_t;
                        L.out_bytes = (uint32_t)Rs;
                        L.gring_bytes = (uint32_t)Rg;
                    }
                }
            }
        }
        if (best >= 0) {
        layout(L.tile);
        for (int b = 0; b < nbr; b++)
            for (int c = b ? P.br_out_end[b - 1] : 0; c < (int)P.br_out_end[b]; c++) {
                const int w = type_width(P.slot[P.out_slot[c]].type);
                P.br_nw[b][w == 1 ? 0 : w == 4 ? 1 : 2]++;
            }
        L.emit = true;
        L.direct = direct_e;
        L.delay = 0;
        return;
        }
        // rows too wide for two staged tiles and a ring in shared memory: the
        // single-stage kernel with its compacted-tile ring in L2 below
    }
    // Scan kernel: S input stages (TMA ring), one scratch tile for computed
    // columns, and a byte ring of R bytes holding compacted tiles until their
    // global offset is resolved (resource budget, §4.3.3).
    const int want_stages = p->o.stages > 0 ? std::min(p->o.stages, kMaxStages) : 0;
    const size_t want_ring = p->o.reserved[0] > 0 ? (size_t)p->o.reserved[0] * 1024 : 0;
    bool ok = false;
    double best_score = -1;
    // compacted-tile ring in global memory (L2-resident) instead of smem
    // default on for compacting chains (measured: frees smem for a third input stage
    // per CTA, C2 2.59 -> 2.29 ms); opts.reserved[6] == 2 keeps the ring in smem
    const bool global_ring = !L.agg && p->o.reserved[6] != 2;
    L.gring_bytes = 0;
    bool direct = !L.agg && nbr == 1;
    for (const HOp &h : ops)
        if (h.kind == K_PRED)
            direct = false;
    L.direct = direct;
    // kernel variants (compute threads NT x rows per thread): 256 x 8 (2048-row tiles),
    // 256 x 4 (1024-row tiles, wide rows); 512 x 4 on request (opts.reserved[4] == 2)
    struct Var { int nt, items; };
    std::vector<Var> vars;
    const int force_items = p->o.reserved[5];              // diagnostics: force rows per thread
    if (!L.agg && p->o.reserved[4] == 2) vars.push_back({512, 4});
    if (!L.agg && p->o.reserved[4] == 3) vars.push_back({512, 8});
    if (L.agg && p->o.reserved[4] != 1 && !agg_mode_for(256))
        vars.push_back({128, 16});   // halves the thread-private partials
    vars.push_back({256, 8});
    if (!L.agg) {
        vars.push_back({256, 6});
        vars.push_back({256, 5});
    }
    vars.push_back({256, 4});
    if (nbr > 1) {   // the branch-loop instance exists for 256 x 8 and 256 x 4
        std::vector<Var> v2;
        for (const Var &v : vars)
            if (v.nt == 256 && (v.items == 8 || v.items == 4)) v2.push_back(v);
        vars = v2;
    }
    // register terminal: 15 (generic) or 18 (narrow sums) compute warps per SM (the aggregate kernel has
    // no writer warps, so its register file takes more compute threads; measured C4
    // 8.56 ms at 256 x 8, 7.43 ms at 384 x 5, 7.06 ms at 448 x 4, 6.52 ms at 480 x 4);
    // opts.reserved[4]: 1 = the 256-thread variants, 4 = 384 x 5, 5 = 448 x 4
    if (L.agg && agg_mode_for(256) == 2 && p->o.reserved[4] != 1) {
        vars.clear();
        // 5 all-64-bit sums with 2 narrow ones: the specialised 544-thread instance
        // (32-bit partials for the narrow sums, 17 compute warps); opts.reserved[4] == 6
        // keeps the generic 480 x 4
        const bool q1shape = P.nagg == 5 && narrow_n == 2 && narrow_all64 &&
                             narrow_flush >= (1 << 16) && p->o.reserved[4] == 0;
        vars.push_back(p->o.reserved[4] == 4 ? Var{384, 5} : p->o.reserved[4] == 5 ? Var{448, 4}
                       : q1shape ? Var{kNarrowNT, kNarrowItems} : Var{480, 4});
    }
    if (force_items > 0) {
        std::vector<Var> v2;
        for (const Var &v : vars)
            if (v.items == force_items) v2.push_back(v);
        if (!v2.empty()) vars = v2;
    }
    for (size_t ii = 0; ii < vars.size(); ii++) {
        const int items = vars[ii].items;
        const int nt = vars[ii].nt;
        const int T = nt * items;
        layout(T);
        size_t W = 0;                       // largest compacted tile (every row survives)
        for (int c = 0; c < P.nout; c++)
            W += (((size_t)T * type_width(P.slot[P.out_slot[c]].type)) + 15) / 16 * 16;
        const size_t agg_bytes = agg_bytes_for(nt);
        const size_t base = scan_ctl_bytes() + P.scratch_bytes + agg_bytes;
        // Candidate (CTAs/SM, input stages, ring bytes) for this variant:
        //  - aggregate: maximise input bytes in flight per SM (no ring);
        //  - no SELECT in the group (every row survives): outputs go straight to their
        //    row offsets, no ring;
        //  - otherwise 2 CTAs/SM x 2 stages when the ring still holds >= 1.9 worst-case
        //    compacted tiles (latency hiding of the compute warps measured best), else
        //    1 CTA/SM with the deepest stage count whose ring holds >= 2.5 tiles.
        struct Cand { int occ, S; size_t Rb, smem; double score; };
        std::vector<Cand> cands;
        for (int occ_t : {4, 3, 2, 1}) {
            if (p->o.ctas_per_sm > 0 ? occ_t != p->o.ctas_per_sm : occ_t > 2) continue;
            const size_t per_cta = std::min(kSmemLimit, (size_t)(228 * 1024) / occ_t - 1024);
            for (int S = 1; S <= 6; S++) {
                if (want_stages && S != want_stages) continue;
                if (base + (size_t)S * P.stage_bytes > per_cta) continue;
                size_t Rb = 0;
                if (!L.agg && !direct && !global_ring) {
                    Rb = want_ring ? want_ring : (per_cta - base - (size_t)S * P.stage_bytes) / 128 * 128;
                    if (Rb < W) continue;
                }
                const size_t smem = base + (size_t)S * P.stage_bytes + Rb;
                if (smem > per_cta) continue;
                if (chain_occupancy(L.agg ? 1 : (nbr > 1 ? 4 : 0), nt, items, smem) < occ_t) continue;
                double inflight = std::min<double>((double)occ_t * S * P.stage_bytes, 192.0 * 1024);
                double score;
                if (L.agg || direct || global_ring) {
                    // (measured: the largest tile wins for the aggregate and the ring, since
                    // the interpreter's per-op dispatch is amortised over the rows per thread)
                    score = inflight + (occ_t == 2 ? 1024.0 : 0) + S + (double)T * 1e4 * ((global_ring || L.agg) ? 1 : 0);
                } else {
                    const double q = (double)Rb / (double)W;
                    const bool ok2 = occ_t == 2 && q >= 1.9 && S >= 2;
                    const bool ok1 = occ_t == 1 && q >= 2.5;
                    // measured (scripts/sweep4.sh): per-tile overhead dominates, so the
                    // largest tile wins before bytes in flight
                    score = (ok2 ? 1e9 : 0) + (ok1 ? 1e8 : 0) + (double)T * 1e4 + inflight + q * 1024.0;
                }
                cands.push_back({occ_t, S, Rb, smem, score});
            }
        }
        // best candidate over all variants (a 2048-row tile with one stage loses to a
        // 1024-row tile with three when the row is wide, e.g. Q1's 38 B + partials)
        for (const Cand &c : cands) {
            const double sc = c.score + (T == 2048 ? 512.0 : 0.0);
            if (!ok || sc > best_score) {
                best_score = sc;
                L.items = items;
                L.nt = nt;
                L.tile = T;
                L.stages = c.S;
                L.ring = 0;
                L.out_bytes = (uint32_t)c.Rb;
                L.smem = c.smem;
                L.ctas = c.occ;
                ok = true;
            }
        }
    }
    if (!ok)
        raise(RW_E_UNSUPPORTED, "fused group exceeds the shared-memory budget");
    layout(L.tile);
    P.agg_mode = agg_mode_for(L.nt);
    // 32-bit partials for the narrow sums (register terminal, kernel variants for
    // (sums, narrow) in {3,4,5} x {1,2}; flush before any could pass 2^32)
    P.agg_narrow = 0;
    bool all64 = true;
    for (int q = 0; q < P.nagg; q++)
        all64 = all64 && (P.agg_type[q] == T_I64 || P.agg_type[q] == T_U64);
    if (P.agg_mode == 2 && all64 && narrow_n >= 1 && narrow_n <= 2 && P.nagg >= 3 && P.nagg <= 5 &&
        p->o.reserved[4] != 1 && narrow_flush >= (1 << 16)) {
        P.agg_narrow = narrow_n;
        P.flush_rows = std::min<int64_t>(P.flush_rows, (int64_t)narrow_flush);
    }
    // the kNarrowNT instance compiles only the 5-sum / 2-narrow / all-64-bit row loop
    if (L.agg && L.nt == kNarrowNT && !(P.nagg == 5 && P.agg_narrow == 2 && all64 && P.agg_mode == 2))
        raise(RW_E_STATE, "internal: Q1-specialised aggregate instance selected for another plan shape");
    // ... and, for exactly the Q1 program shape, the fused row path (agg_tile_q1):
    // SELECT on an i32 stage column vs a constant, then two i64 fixed-point factors
    // d = a * (k -/+ b), c = d * (k -/+ e) over stage columns, summed as the last two of
    // [narrow, narrow, wide stage column, d, c].  opts.reserved[7] == 2 keeps the interpreter.
    P.q1fused = 0;
    if (L.agg && L.nt == kNarrowNT && P.nops == 3 && p->o.reserved[7] != 2) {
        const DevOp &o0 = P.ops[0], &o1 = P.ops[1], &o2 = P.ops[2];
        const uint8_t mulaff = (uint8_t)(64 + T_I64 * 8 + E_MULAFF);
        auto stage_loc = [](uint32_t loc) { return (loc & kLocScratch) == 0; };
        const bool ok = o0.kind == K_PRED && o0.code < 64 && (o0.code >> 3) == T_I32 && stage_loc(o0.a) &&
                        o1.kind == K_EXPR && o1.code == mulaff && o2.kind == K_EXPR && o2.code == mulaff &&
                        o1.ta == T_I64 && (o1.tb & 0x7f) == T_I64 && o2.ta == T_I64 && (o2.tb & 0x7f) == T_I64 &&
                        stage_loc(o1.a) && stage_loc(o1.b) && stage_loc(o2.b) && o2.a == o1.dst &&
                        P.agg_loc[3] == o1.dst && P.agg_loc[4] == o2.dst && stage_loc(P.agg_loc[0]) &&
                        stage_loc(P.agg_loc[1]) && stage_loc(P.agg_loc[2]);
        bool gstage = true;
        for (int c = 0; c < P.ngc; c++)
            gstage = gstage && stage_loc(P.g_loc[c]);
        P.q1fused = ok && gstage ? 1 : 0;
    }
    if (global_ring && !L.direct) {
        size_t W = 0;
        for (int c = 0; c < P.nout; c++)
            W += (((size_t)L.tile * type_width(P.slot[P.out_slot[c]].type)) + 15) / 16 * 16;
        L.gring_bytes = (uint32_t)std::max<size_t>(want_ring ? want_ring : 128 * 1024, 4 * W);
        L.out_bytes = L.gring_bytes;
    }
}

// ---------------------------------------------------------------------------
// Algorithm 2 analogue (§4.2, §4.3.3; reading A20): operators are
// fused greedily, earliest first, while the group's kernel fits its resource budget
// (micro-ops, tile columns, shared memory); a group that does not fit is split after
// its longest fitting prefix, whose output is then materialised, and the grouping is
// rebuilt.  A single operator that does not fit is an error (RW_E_UNSUPPORTED).
// ---------------------------------------------------------------------------
bool lowers(rw_plan *p, const Group &g)
{
    try {
        Lowered L;
        lower(p, g, g.kind == G_SCAN ? p->nodes[g.source].types : join_src_types(p, g), L);
        return true;
    } catch (const RwError &e) {
        if (e.s != RW_E_UNSUPPORTED)
            throw;
        return false;
    }
}

Grouping build_groups(const rw_plan *p_, int out_node)
{
    rw_plan *p = const_cast<rw_plan *>(p_);
    std::vector<int> cuts;
    for (int iter = 0;; iter++) {
        Grouping G = build_groups_once(p, out_node, cuts);
        if (!p->o.fuse || iter > (int)p->nodes.size())
            return G;
        int cut = -1;
        for (const Group &g : G.groups) {
            if (g.kind == G_SET || lowers(p, g))
                continue;
            const std::vector<int> &c = g.chain;
            const int k = (int)c.size();
            if (g.kind == G_SCAN) {
                for (int m = k; m >= 1 && cut < 0; m--) {
                    Group h = g;
                    h.chain.assign(c.begin(), c.begin() + m);
                    h.agg = -1;
                    h.out = c[m - 1];
                    if (lowers(p, h))
                        cut = c[m - 1];
                }
            } else {
                for (int m = k; m >= 0 && cut < 0; m--) {
                    Group h = g;
                    h.chain.assign(c.begin(), c.begin() + m);
                    h.agg = -1;
                    h.out = m > 0 ? c[m - 1] : g.join;
                    if (lowers(p, h))
                        cut = m > 0 ? c[m - 1] : g.join;
                }
                if (cut < 0) {
                    // the expansion alone does not fit: materialise an upstream pre-chain, else
                    // the inner JOIN of a 3-input group
                    int best = -1;
                    for (int sd = 0; sd < 3; sd++)
                        if (!g.prechain[sd].empty() && (best < 0 || g.prechain[sd].size() > g.prechain[best].size()))
                            best = sd;
                    if (best >= 0) cut = g.prechain[best].back();
                    else if (g.join_in >= 0) cut = g.join_in;
                }
            }
            if (cut < 0 || std::find(cuts.begin(), cuts.end(), cut) != cuts.end()) {
                Lowered L;   // rethrows the budget error of the group that cannot be split
                lower(p, g, g.kind == G_SCAN ? p->nodes[g.source].types : join_src_types(p, g), L);
            }
            break;
        }
        if (cut < 0)
            return G;
        cuts.push_back(cut);
    }
}

// ---------------------------------------------------------------------------
// Execution
// ---------------------------------------------------------------------------
struct ExecCtx {
    rw_plan *p;
    const rw_relation_in *in;
    int nin;
    Grouping G;
    std::vector<Rel> rels;             // per group output
    std::vector<char> done;
    int final_group;
    rw_relation_out *out;
    int64_t *final_n_dev;
};

Rel input_rel(ExecCtx &X, int node)
{
    const Node &n = X.p->nodes[node];
    const rw_relation_in &ri = X.in[n.input_index];
    Rel r;
    r.types = n.types;
    for (size_t c = 0; c < n.types.size(); c++)
        r.cols.push_back(ri.cols[c]);
    r.n_host = ri.n;
    r.cap = ri.n;
    return r;
}

Rel rel_of(ExecCtx &X, int node)
{
    if (X.p->nodes[node].kind == N_INPUT)
        return input_rel(X, node);
    return X.rels[X.G.produced_by.at(node)];
}

int64_t host_count(ExecCtx &X, const Rel &r)
{
    if (r.n_host >= 0)
        return r.n_host;
    rw_plan *p = X.p;
    cuda_check(cudaMemcpyAsync(p->jtot_host + 2, r.n_dev, 8, cudaMemcpyDeviceToHost, p->stream), "copy count");
    cuda_check(cudaStreamSynchronize(p->stream), "sync");
    return p->jtot_host[2];
}

void make_output(ExecCtx &X, int gi, const std::vector<int> &types, int64_t cap, Rel &o, std::vector<void *> &outp,
                 int64_t &capacity, int64_t *&n_dev)
{
    rw_plan *p = X.p;
    o.types = types;
    outp.clear();
    if (gi == X.final_group) {
        for (size_t c = 0; c < types.size(); c++)
            outp.push_back(X.out->cols[c]);
        capacity = X.out->capacity;
        n_dev = X.final_n_dev;
    } else {
        for (int t : types)
            outp.push_back(temp_alloc(p, (size_t)std::max<int64_t>(cap, 1) * type_width(t)));
        capacity = cap;
        n_dev = p->cnt + gi;
    }
    for (void *q : outp)
        o.cols.push_back(q);
    o.n_dev = n_dev;
    o.cap = std::min(cap, capacity);
}

unsigned long long *agg_buffer(rw_plan *p, int node, size_t words)
{
    auto it = p->agg_acc.find(node);
    if (it != p->agg_acc.end())
        return it->second;
    unsigned long long *b = (unsigned long long *)dev_alloc(p, words * 8);
    cuda_check(cudaMemsetAsync(b, 0, words * 8, p->stream), "memset agg");
    p->agg_acc[node] = b;
    return b;
}

// order-preserving key images of a relation's leading nkey columns (join2.cu KeySrc)
KeySrc key_src(const Rel &r, int nkey)
{
    KeySrc k{};
    k.ncol = nkey;
    for (int c = 0; c < nkey; c++) {
        k.col[c] = r.cols[c];
        k.type[c] = (uint8_t)r.types[c];
    }
    return k;
}

// image of a key constant (for key SELECTs fused into the matching): as col_img
uint64_t key_const_img(int type, int64_t v)
{
    const uint64_t u = (uint64_t)wrap_to(type, v);
    switch (type) {
    case T_I32: return (uint32_t)u ^ 0x80000000u;
    case T_U32: return (uint32_t)u;
    case T_I64: return u ^ 0x8000000000000000ull;
    case T_U64: return u;
    default: return (uint8_t)u;
    }
}

// JOIN group (2 or 3 inputs): single-pass run matching (chained for 3 inputs), tile
// index, fused expansion.  No host synchronisation when the group writes the caller's
// output (its capacity is given); a materialised join intermediate reads its row count.
void run_join_group(ExecCtx &X, int gi, const Group &g, Rel &o, std::vector<void *> &outp, int64_t &capacity,
                    int64_t *&n_dev)
{
    rw_plan *p = X.p;
    const Node &jn = p->nodes[g.join];
    const Node &outn = p->nodes[g.out];
    const bool three = g.join_in >= 0;
    const int nkey = jn.nkey;
    Rel ra = rel_of(X, g.jl), rb = rel_of(X, g.jr);
    Rel rc;
    if (three) rc = rel_of(X, g.jc);
    const int64_t na = host_count(X, ra), nb = host_count(X, rb), nc = three ? host_count(X, rc) : 0;
    // run records and the expansion hold 32-bit row indices
    if (na > (int64_t)UINT32_MAX || nb > (int64_t)UINT32_MAX || nc > (int64_t)UINT32_MAX)
        raise(RW_E_UNSUPPORTED, "join input above 2^32 rows per GPU (materialised intermediate): shard across ranks");
    int kbytes = 0;
    for (int c = 0; c < nkey; c++)
        kbytes += type_width(ra.types[c]) == 8 ? 8 : 4;
    if (kbytes > 8)
        raise(RW_E_UNSUPPORTED, "join keys wider than 8 bytes (nkey = 2 needs 32-bit key columns)");
    const bool wide = kbytes > 4;
    const int mt = match_partition();
    // ---- run matching ----
    auto status_at = [&](int64_t words) {
        uint64_t *st = p->status + p->status_used;
        p->status_used += words;
        return st;
    };
    const int64_t nparts1 = (na + nb + mt - 1) / mt;
    const int64_t cap1 = std::max<int64_t>(1, std::min(na, nb));
    const int64_t nparts2 = three ? (cap1 + nc + mt - 1) / mt : 0;
    const int64_t cap2 = three ? std::max<int64_t>(1, std::min(cap1, nc)) : 0;
    const int T = 0;   // set below from the lowering
    (void)T;
    Lowered L;
    lower(p, g, join_src_types(p, g), L);
    const int64_t T2 = L.tile;
    const double maxc = three ? (double)na * (double)nb * (double)nc : (double)na * (double)nb;
    // tile index capacity: every candidate when that is below 2^34 (no host sync), else
    // the exact count after a synchronisation
    const bool exact_tiles = maxc > 17179869184.0;
    p->status_used = 0;
    int64_t status_need = 2 * (nparts1 + 1) + 2 * (nparts2 + 1) + 16;
    int64_t cap_tiles = exact_tiles ? 0 : (int64_t)(maxc / (double)T2) + 2;
    ensure_status(p, status_need + cap_tiles + 1);
    auto mk_u32 = [&](int64_t n) { return (uint32_t *)temp_alloc(p, (size_t)(n + 8) * 4); };
    auto mk_u64 = [&](int64_t n) { return (uint64_t *)temp_alloc(p, (size_t)(n + 8) * 8); };
    int64_t *tot1 = p->jtot, *tot2 = p->jtot + 2;
    cuda_check(cudaMemsetAsync(p->jtot, 0, 32, p->stream), "memset totals");
    MatchLaunch M{};
    M.A = key_src(ra, nkey);
    M.B = key_src(rb, nkey);
    M.nA = na;
    M.nB = nb;
    M.nparts = nparts1;
    M.split = (int64_t *)temp_alloc(p, (size_t)(nparts1 + 1) * 8);
    M.cap_runs = cap1;
    M.s0 = mk_u32(cap1);
    M.s1 = mk_u32(cap1);
    M.len1 = mk_u32(cap1);
    M.off = mk_u64(cap1);
    if (three) {
        M.key_out = temp_alloc(p, (size_t)(cap1 + 8) * (wide ? 8 : 4));
        M.w_out = mk_u64(cap1);
    }
    M.st_runs = status_at(nparts1 + 1);
    M.st_cands = status_at(nparts1 + 1);
    M.ep_runs = next_epoch(p);
    M.ep_cands = next_epoch(p);
    M.ctrs = p->ctrs;
    M.totals = tot1;
    for (int sid : g.pre)
        for (const rw_pred &a : p->nodes[sid].preds) {
            if (nkey != 1)
                raise(RW_E_STATE, "internal: key SELECT fused into a multi-column key");
            M.kop[M.nkpred] = (uint8_t)a.op;
            M.kpk[M.nkpred] = key_const_img(ra.types[0], a.rhs_const);
            M.nkpred++;
        }
    cuda_check(match_launch(M, wide, p->stream), "k_jmatch");
    p->launches += nparts1 > 0 ? 2 : 1;
    JoinEmit XJ{};
    const int64_t *totals = tot1;
    if (three) {
        MatchLaunch M2{};
        M2.A.img = M.key_out;
        M2.A.ncol = 1;
        M2.B = key_src(rc, nkey);
        M2.nA = cap1;
        M2.nA_dev = tot1;                    // first-level runs (device)
        M2.nB = nc;
        M2.nparts = nparts2;
        M2.split = (int64_t *)temp_alloc(p, (size_t)(nparts2 + 1) * 8);
        M2.wA = M.w_out;
        M2.chain1 = 1;
        M2.c_s0 = M.s0;
        M2.c_s1 = M.s1;
        M2.c_len1 = M.len1;
        M2.cap_runs = cap2;
        M2.s0 = mk_u32(cap2);
        M2.s1 = mk_u32(cap2);
        M2.len1 = mk_u32(cap2);
        M2.s2 = mk_u32(cap2);
        M2.len2 = mk_u32(cap2);
        M2.off = mk_u64(cap2);
        M2.st_runs = status_at(nparts2 + 1);
        M2.st_cands = status_at(nparts2 + 1);
        M2.ep_runs = next_epoch(p);
        M2.ep_cands = next_epoch(p);
        M2.ctrs = p->ctrs;
        M2.totals = tot2;
        cuda_check(match_launch(M2, wide, p->stream), "k_jmatch (chained)");
        p->launches += nparts2 > 0 ? 2 : 1;
        XJ.off = M2.off;
        XJ.s0 = M2.s0;
        XJ.s1 = M2.s1;
        XJ.len1 = M2.len1;
        XJ.s2 = M2.s2;
        XJ.len2 = M2.len2;
        totals = tot2;
    } else {
        XJ.off = M.off;
        XJ.s0 = M.s0;
        XJ.s1 = M.s1;
        XJ.len1 = M.len1;
    }
    // ---- output: the caller's (capacity given) or a materialised intermediate ----
    int64_t total_host = -1;
    if (gi != X.final_group || exact_tiles) {
        cuda_check(cudaMemcpyAsync(p->jtot_host, totals, 16, cudaMemcpyDeviceToHost, p->stream), "copy totals");
        cuda_check(cudaStreamSynchronize(p->stream), "sync after join runs");
        total_host = p->jtot_host[1];
        if (exact_tiles)
            cap_tiles = (total_host + T2 - 1) / T2 + 2;
    }
    if (exact_tiles)
        ensure_status(p, p->status_used + cap_tiles + 1);
    make_output(X, gi, outn.types, gi == X.final_group ? X.out->capacity : (L.agg ? p->nodes[g.agg].D : total_host), o,
                outp, capacity, n_dev);
    // ---- tile index ----
    int64_t *tile_run = (int64_t *)temp_alloc(p, (size_t)std::max<int64_t>(cap_tiles, 2) * 8);
    int32_t *ovf = (int32_t *)(p->err + 8);
    cuda_check(jtiles_launch(XJ.off, totals, T2, cap_tiles, tile_run, ovf, p->sms, p->stream), "k_jtiles");
    p->launches++;
    // ---- expansion fused with the downstream chain ----
    XJ.tile_run = tile_run;
    XJ.rec_cap4 = join_rec_cap4((int)T2);
    XJ.rec_stage_bytes = (uint32_t)join_rec_stage_bytes(three ? 3 : 2, (int)T2);
    // input slot -> (input, raw column): the slot space is A's, B's[, C's] columns side by side
    const int nac = (int)ra.types.size(), nbc = (int)rb.types.size();
    XJ.ncols = L.P.nin;
    for (int i = 0; i < L.P.nin; i++) {
        const int c = L.in_src[i];
        int side, col;
        if (c < nac) { side = 0; col = c; }
        else if (c < nac + nbc) { side = 1; col = c - nac; }
        else { side = 2; col = c - nac - nbc; }
        const Rel &src = side == 0 ? ra : side == 1 ? rb : rc;
        XJ.src[i] = src.cols[col];
        XJ.side[i] = (uint8_t)side;
        XJ.w[i] = (uint8_t)type_width(src.types[col]);
    }
    XJ.regpath = XJ.ncols <= 4;
    for (int i = 0; i < XJ.ncols; i++)
        if (XJ.w[i] == 8) XJ.regpath = 0;
    if (p->o.reserved[6] == 6) XJ.regpath = 0;        // diagnostics: cp.async gathers
    for (size_t c = 0; c < outp.size(); c++)
        L.P.out_ptr[c] = outp[c];
    L.P.out_capacity = capacity;
    TileLaunch TL{};
    TL.n_ptr = totals + 1;
    TL.stages = L.stages;
    TL.epoch = next_epoch(p);
    TL.status = status_at(cap_tiles + 1);
    TL.ctrs = p->ctrs;
    TL.n_dev = n_dev;
    TL.err = p->err;
    TL.out_bytes = L.out_bytes;
    TL.dbg = p->o.reserved[1];
    const int grid = p->sms * L.ctas;
    unsigned long long *acc = nullptr;
    if (L.agg) {
        const size_t words = (size_t)p->nodes[g.agg].D * (L.P.nagg + 1) * 2;
        acc = agg_buffer(p, g.agg, words);
        TL.agg_acc = acc;
    }
    cuda_check(join_emit_launch(L.P, TL, XJ, L.nt, L.items, three ? 3 : 2, L.smem, grid, p->stream), "k_join_emit");
    p->launches++;
    if (L.agg) {
        L.F.acc = acc;
        L.F.acc_w = acc;
        for (size_t c = 0; c < outp.size(); c++)
            L.F.out[c] = outp[c];
        L.F.capacity = capacity;
        L.F.n_dev = n_dev;
        L.F.err = p->err;
        cuda_check(agg_finalize_launch(L.F, p->stream), "k_agg_finalize");
        p->launches++;
    }
}

void run_group(ExecCtx &X, int gi)
{
    if (X.done[gi])
        return;
    const Group &g = X.G.groups[gi];
    for (int d : g.deps)
        run_group(X, d);
    rw_plan *p = X.p;
    const Node &outn = p->nodes[g.out];
    Rel o;
    std::vector<void *> outp;
    int64_t capacity = 0;
    int64_t *n_dev = nullptr;

    if (g.kind == G_SCAN && !p->o.fuse && p->o.zero_copy_project && g.agg < 0 && g.chain.size() == 1 &&
        gi != X.final_group && p->nodes[g.chain[0]].kind == N_PROJECT) {
        // operator-at-a-time variant with a zero-copy PROJECT: alias plain column references
        const Node &pn = p->nodes[g.chain[0]];
        bool plain = true;
        for (int r : pn.roots)
            plain = plain && pn.exprs[r].op == RW_COL && pn.exprs[r].type == p->nodes[pn.in].types[pn.exprs[r].a];
        if (plain) {
            Rel src = rel_of(X, g.source);
            o = src;
            o.types = pn.types;
            o.cols.clear();
            for (int r : pn.roots)
                o.cols.push_back(src.cols[pn.exprs[r].a]);
            X.rels[gi] = o;
            X.done[gi] = 1;
            return;
        }
    }
    if (g.kind == G_SCAN) {
        Rel src = rel_of(X, g.source);
        Lowered L;
        lower(p, g, src.types, L);
        const int T = L.tile;
        int64_t cap_out = L.agg ? p->nodes[g.agg].D : src.cap;
        make_output(X, gi, outn.types, cap_out, o, outp, capacity, n_dev);
        bool aligned = true;
        for (int i = 0; i < L.P.nin; i++) {
            L.P.in_ptr[i] = src.cols[L.in_src[i]];
            if (((uintptr_t)L.P.in_ptr[i]) & 15)
                aligned = false;
        }
        const int64_t max_tiles = (src.cap + T - 1) / T;
        ensure_status(p, max_tiles + 1);
        TileLaunch TL{};
        TL.n = src.n_host >= 0 ? src.n_host : 0;
        TL.n_ptr = src.n_host >= 0 ? nullptr : src.n_dev;
        TL.stages = L.stages;
        TL.dbg = p->o.reserved[1];
        TL.dbg_ts = (uint64_t *)(((uint64_t)(uint32_t)p->o.reserved[3] << 32) | (uint32_t)p->o.reserved[2]);
        TL.out_bytes = L.out_bytes;
        TL.direct = L.direct ? 1 : 0;
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(max_tiles, (int64_t)p->sms * L.ctas));
        if (L.gring_bytes) {
            const size_t need = (size_t)grid * L.gring_bytes;
            if (need > p->gring_cap) {
                if (p->gring) cudaFreeAsync(p->gring, p->stream);
                p->gring = (char *)dev_alloc(p, need);
                p->gring_cap = need;
            }
            TL.gring = p->gring;
            TL.gring_bytes = L.gring_bytes;
        }
        TL.use_tma = aligned ? 1 : 0;
        TL.epoch = next_epoch(p);
        TL.status = p->status;
        TL.ctrs = p->ctrs;
        TL.err = p->err;
        if (L.agg) {
            const Node &an = p->nodes[g.agg];
            const size_t words = (size_t)an.D * (L.P.nagg + 1) * 2;
            unsigned long long *acc = agg_buffer(p, g.agg, words);
            TL.agg_acc = acc;
            TL.n_dev = n_dev;
            cuda_check(scan_chain_launch(L.P, TL, true, L.nt, L.items, L.smem, grid, p->stream), "k_scan_chain<agg>");
            p->launches++;
            L.F.acc = acc;
            L.F.acc_w = acc;
            for (size_t c = 0; c < outp.size(); c++)
                L.F.out[c] = outp[c];
            L.F.capacity = capacity;
            L.F.n_dev = n_dev;
            L.F.err = p->err;
            if (!p->defer_finalize) {
                cuda_check(agg_finalize_launch(L.F, p->stream), "k_agg_finalize");
                p->launches++;
            }
        } else {
            for (size_t c = 0; c < outp.size(); c++)
                L.P.out_ptr[c] = outp[c];
            L.P.out_capacity = capacity;
            TL.n_dev = n_dev;
            if (L.emit) {
                TL.delay = L.delay;
                cuda_check(scan_emit_launch(L.P, TL, L.nt, L.items, L.smem, grid, p->stream, L.teams), "k_scan_emit");
            } else {
                cuda_check(scan_chain_launch(L.P, TL, false, L.nt, L.items, L.smem, grid, p->stream), "k_scan_chain");
            }
            p->launches++;
        }
    } else if (g.kind == G_SET) {
        const Node &sn = p->nodes[g.join];
        Rel xr = rel_of(X, sn.left), yr = rel_of(X, sn.right);
        const int64_t nx = host_count(X, xr), ny = host_count(X, yr);
        const int64_t cap = sn.setop == RW_UNION ? nx + ny : sn.setop == RW_INTERSECT ? std::min(nx, ny) : nx;
        make_output(X, gi, outn.types, cap, o, outp, capacity, n_dev);
        SetLaunch S{};
        S.ncols = (int)sn.types.size();
        S.op = sn.setop == RW_UNION ? 0 : sn.setop == RW_INTERSECT ? 1 : 2;
        for (int c = 0; c < S.ncols; c++) {
            S.types[c] = (uint8_t)sn.types[c];
            S.x[c] = xr.cols[c];
            S.y[c] = yr.cols[c];
            S.out[c] = outp[c];
        }
        S.nx = nx;
        S.ny = ny;
        S.nparts = (nx + ny + set_partition_rows() - 1) / set_partition_rows();
        S.cap = capacity;
        S.split = (int64_t *)temp_alloc(p, (size_t)(S.nparts + 1) * 8);
        S.pcount = (uint64_t *)temp_alloc(p, (size_t)(S.nparts + 1) * 8);
        S.nbr = (int32_t *)temp_alloc(p, (size_t)(S.nparts + 1) * 4);
        S.total = n_dev;
        // one pass with a decoupled look-back over the partitions (opts.reserved[1] & 1:
        // the count / scan / write passes)
        if (!(p->o.reserved[1] & 1)) {
            ensure_status(p, S.nparts + 1);
            S.status = p->status;
            S.epoch = next_epoch(p);
            S.ctrs = p->ctrs;
        }
        cuda_check(set_op_launch(S, p->sms, p->stream), "k_set_op");
        p->launches += S.status ? (S.nparts > 0 ? 2 : 1) : (S.nparts > 0 ? 4 : 2);
    } else {
        run_join_group(X, gi, g, o, outp, capacity, n_dev);
    }
    X.rels[gi] = o;
    X.done[gi] = 1;
}

std::vector<int> &schema_types(rw_plan *p, int node) { return p->nodes[node].types; }

// errors an aggregate finalisation recorded (err[1], err[3] copied to jtot_host + 8)
void raise_agg_errors(rw_plan *p)
{
    const int32_t *e = (const int32_t *)(p->jtot_host + 8);
    if (e[1])
        raise(RW_E_DOMAIN, std::to_string(e[1]) + " rows had a group value outside its domain");
    if (e[3])
        raise(RW_E_DOMAIN, std::to_string(e[3]) + " tiles held a summed value outside its declared [lo, hi] "
                                                  "bounds (rw_plan_add_input): the 32-bit partials are not exact");
}

void check_inputs(rw_plan *p, const rw_relation_in *in, int nin)
{
    if (nin != (int)p->inputs.size())
        raise(RW_E_ARG, "expected " + std::to_string(p->inputs.size()) + " input relations, got " + std::to_string(nin));
    for (int i = 0; i < nin; i++) {
        if (in[i].n < 0)
            raise(RW_E_ARG, "negative row count");
        if (in[i].n > (int64_t)UINT32_MAX)
            raise(RW_E_UNSUPPORTED, "relations above 2^32 rows per GPU: shard across ranks");
        if (in[i].n > 0 && !in[i].cols)
            raise(RW_E_ARG, "null column array");
    }
}

void execute(rw_plan *p, const rw_relation_in *in, int nin, int out_node, rw_relation_out *out)
{
    node_at(p, out_node);
    if (!out || (!out->cols && out->capacity > 0))
        raise(RW_E_ARG, "null output");
    check_inputs(p, in, nin);
    cuda_check(cudaSetDevice(p->o.device), "cudaSetDevice");
    p->launches = 0;
    if (p->nodes[out_node].kind == N_INPUT)
        raise(RW_E_UNSUPPORTED, "output node is an input relation");
    ExecCtx X;
    X.p = p;
    X.in = in;
    X.nin = nin;
    X.G = build_groups(p, out_node);
    X.rels.resize(X.G.groups.size());
    X.done.assign(X.G.groups.size(), 0);
    X.final_group = X.G.produced_by.at(out_node);
    X.out = out;
    if ((int)X.G.groups.size() + 1 > p->cnt_cap) {
        if (p->cnt) cudaFreeAsync(p->cnt, p->stream);
        p->cnt_cap = (int)X.G.groups.size() + 8;
        p->cnt = (int64_t *)dev_alloc(p, (size_t)p->cnt_cap * 8);
    }
    X.final_n_dev = out->n_dev ? out->n_dev : p->cnt + (p->cnt_cap - 1);
    try {
        run_group(X, X.final_group);
    } catch (...) {
        free_temps(p);
        throw;
    }
    free_temps(p);
    out->n = -1;
    if (!out->n_dev) {
        cuda_check(cudaMemcpyAsync(p->jtot_host + 2, X.final_n_dev, 8, cudaMemcpyDeviceToHost, p->stream), "copy n");
        cuda_check(cudaMemcpyAsync(p->jtot_host + 8, p->err, 16, cudaMemcpyDeviceToHost, p->stream), "copy err");
        cuda_check(cudaStreamSynchronize(p->stream), "sync");
        out->n = p->jtot_host[2];
        raise_agg_errors(p);
        if (out->n > out->capacity)
            raise(RW_E_CAPACITY, "output needs " + std::to_string(out->n) + " rows, capacity " +
                                     std::to_string(out->capacity));
    }
}

// Input-dependence fusion (§4.4, Fig. 14(d)): the SELECT / PROJECT chains from
// one common INPUT to each requested node become the branches of one scan group.
void execute_multi(rw_plan *p, const rw_relation_in *in, int nin, const int32_t *nodes, int nout,
                   rw_relation_out *outs)
{
    if (nout <= 0 || !nodes || !outs)
        raise(RW_E_ARG, "execute_multi: no outputs");
    for (int k = 0; k < nout; k++) {
        node_at(p, nodes[k]);
        if (!outs[k].cols && outs[k].capacity > 0)
            raise(RW_E_ARG, "null output");
    }
    check_inputs(p, in, nin);
    cuda_check(cudaSetDevice(p->o.device), "cudaSetDevice");
    std::vector<std::vector<int>> chains(nout);
    int src = -1;
    bool fusable = p->o.fuse && nout > 1 && nout <= kMaxBranch;
    for (int k = 0; k < nout && fusable; k++) {
        int cur = nodes[k];
        while (is_unary_chain(p->nodes[cur].kind)) {
            chains[k].insert(chains[k].begin(), cur);
            cur = p->nodes[cur].in;
        }
        if (chains[k].empty() || p->nodes[cur].kind != N_INPUT || (src >= 0 && cur != src))
            fusable = false;
        src = cur;
    }
    if (!fusable) {
        int64_t launches = 0;
        for (int k = 0; k < nout; k++) {
            execute(p, in, nin, nodes[k], &outs[k]);
            launches += p->launches;
        }
        p->launches = launches;
        return;
    }
    p->launches = 0;
    Group g;
    g.kind = G_SCAN;
    g.source = src;
    g.out = nodes[0];
    g.branches = chains;
    const Node &sn = p->nodes[src];
    Lowered L;
    lower(p, g, sn.types, L);
    const rw_relation_in &ri = in[sn.input_index];
    const int T = L.tile;
    bool aligned = true;
    for (int i = 0; i < L.P.nin; i++) {
        L.P.in_ptr[i] = ri.cols[L.in_src[i]];
        if (((uintptr_t)L.P.in_ptr[i]) & 15)
            aligned = false;
    }
    if (p->cnt_cap < nout + 1) {
        if (p->cnt) cudaFreeAsync(p->cnt, p->stream);
        p->cnt_cap = nout + 8;
        p->cnt = (int64_t *)dev_alloc(p, (size_t)p->cnt_cap * 8);
    }
    int c = 0;
    for (int k = 0; k < nout; k++) {
        const int ncol = (int)p->nodes[nodes[k]].types.size();
        if (L.P.br_out_end[k] != c + ncol)
            raise(RW_E_ARG, "execute_multi: branch schema mismatch");
        for (int q = 0; q < ncol; q++)
            L.P.out_ptr[c + q] = outs[k].cols[q];
        c += ncol;
        L.P.br_cap[k] = outs[k].capacity;
    }
    L.P.out_capacity = outs[0].capacity;
    const int64_t max_tiles = (ri.n + T - 1) / T;
    ensure_status(p, (int64_t)nout * (max_tiles + 1));
    TileLaunch TL{};
    TL.n = ri.n;
    TL.stages = L.stages;
    TL.dbg = p->o.reserved[1] & ~4;
    TL.out_bytes = L.out_bytes;
    TL.direct = 0;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(max_tiles, (int64_t)p->sms * L.ctas));
    if (L.gring_bytes) {
        const size_t need = (size_t)grid * L.gring_bytes;
        if (need > p->gring_cap) {
            if (p->gring) cudaFreeAsync(p->gring, p->stream);
            p->gring = (char *)dev_alloc(p, need);
            p->gring_cap = need;
        }
        TL.gring = p->gring;
        TL.gring_bytes = L.gring_bytes;
    }
    TL.use_tma = aligned ? 1 : 0;
    TL.epoch = next_epoch(p);
    TL.status = p->status;
    TL.status_stride = max_tiles + 1;
    TL.ctrs = p->ctrs;
    TL.err = p->err;
    for (int k = 0; k < nout; k++) {
        int64_t *nd = outs[k].n_dev ? outs[k].n_dev : p->cnt + k;
        if (k == 0) TL.n_dev = nd;
        else TL.br_n_dev[k] = nd;
    }
    if (L.emit) {
        TL.delay = L.delay;
        cuda_check(scan_emit_launch(L.P, TL, L.nt, L.items, L.smem, grid, p->stream), "k_scan_emit<multi>");
    } else {
        cuda_check(scan_chain_launch(L.P, TL, false, L.nt, L.items, L.smem, grid, p->stream), "k_scan_chain<multi>");
    }
    p->launches++;
    bool any_sync = false;
    for (int k = 0; k < nout; k++)
        if (!outs[k].n_dev) {
            cuda_check(cudaMemcpyAsync(p->jtot_host + 4 + k, p->cnt + k, 8, cudaMemcpyDeviceToHost, p->stream),
                       "copy n");
            any_sync = true;
        }
    if (any_sync)
        cuda_check(cudaStreamSynchronize(p->stream), "sync");
    for (int k = 0; k < nout; k++) {
        outs[k].n = -1;
        if (outs[k].n_dev)
            continue;
        outs[k].n = p->jtot_host[4 + k];
        if (outs[k].n > outs[k].capacity)
            raise(RW_E_CAPACITY, "output " + std::to_string(k) + " needs " + std::to_string(outs[k].n) +
                                     " rows, capacity " + std::to_string(outs[k].capacity));
    }
}

// Host-streamed execution (the paper's PCIe experiment P:241-252):
// a plan that is one scan group over one INPUT relation runs over row chunks.  The
// H2D copy of chunk k+1 (copy stream), the fused kernel of chunk k (plan stream) and
// the D2H copy of chunk k-1's compacted output (second copy stream) overlap; only
// compacted rows cross PCIe back.  Chunk outputs are appended in chunk order, so the
// result equals rw_plan_execute over the whole relation (row order included).  An
// aggregate accumulates every chunk in its 128-bit accumulators and finalises once.
// Returns false when the plan does not have that shape (the caller copies whole).
bool execute_host_streamed(rw_plan *p, const rw_relation_in *in, int nin, int out_node, rw_relation_out *out)
{
    node_at(p, out_node);
    if (p->nodes[out_node].kind == N_INPUT)
        return false;
    Grouping G = build_groups(p, out_node);
    if (G.groups.size() != 1)
        return false;
    const Group &g = G.groups[0];
    if (g.kind != G_SCAN || p->nodes[g.source].kind != N_INPUT)
        return false;
    const Node &sn = p->nodes[g.source];
    const rw_relation_in &ri = in[sn.input_index];
    const int lg = p->o.host_chunk_log2 > 0 ? std::min(p->o.host_chunk_log2, 31) : 25;
    const int64_t C = (int64_t)1 << lg;
    if (ri.n <= C)
        return false;
    const bool agg = g.agg >= 0;
    const Node &on = p->nodes[out_node];
    const int nci = (int)sn.types.size(), nco = (int)on.types.size();
    const int64_t ocap = agg ? on.D : C;
    const int64_t nch = (ri.n + C - 1) / C;
    auto &H = p->hs;
    if (!H.init) {
        cuda_check(cudaStreamCreateWithFlags(&H.sh, cudaStreamNonBlocking), "stream");
        cuda_check(cudaStreamCreateWithFlags(&H.sd, cudaStreamNonBlocking), "stream");
        for (int a = 0; a < 4; a++)
            for (int b = 0; b < 2; b++)
                cuda_check(cudaEventCreateWithFlags(&H.ev[a][b], cudaEventDisableTiming), "event");
        cuda_check(cudaMallocHost(&H.hcnt, 2 * sizeof(int64_t)), "cudaMallocHost");
        H.init = true;
    }
    cudaStream_t sh = H.sh, sd = H.sd;
    cudaEvent_t *ev_h2d = H.ev[0], *ev_in_free = H.ev[1], *ev_cnt = H.ev[2], *ev_out_free = H.ev[3];
    int64_t *hcnt = H.hcnt;
    // chunk buffers: 2 x (input columns, output columns, count), one allocation
    size_t per = 0;
    for (int c = 0; c < nci; c++) per += ((size_t)C * type_width(sn.types[c]) + 255) / 256 * 256;
    for (int c = 0; c < nco; c++) per += ((size_t)ocap * type_width(on.types[c]) + 255) / 256 * 256;
    per += 256;                                         // count; per stays a multiple of 256
    if (2 * per > H.bytes) {
        cuda_check(cudaStreamSynchronize(p->stream), "sync");
        if (H.buf) cudaFree(H.buf);
        H.buf = nullptr;
        H.bytes = 0;
        cudaError_t e = cudaMalloc(&H.buf, 2 * per);
        if (e == cudaErrorMemoryAllocation)
            raise(RW_E_OOM, "host-streamed chunk buffers: out of device memory");
        cuda_check(e, "cudaMalloc");
        H.bytes = 2 * per;
    }
    auto cleanup = [&]() {
        cudaStreamSynchronize(sh);
        cudaStreamSynchronize(sd);
        cudaStreamSynchronize(p->stream);
        p->defer_finalize = false;
    };
    try {
        std::vector<void *> ib[2], ob[2];
        int64_t *nd[2];
        for (int b = 0; b < 2; b++) {
            char *q = H.buf + b * per;
            for (int c = 0; c < nci; c++) {
                ib[b].push_back(q);
                q += ((size_t)C * type_width(sn.types[c]) + 255) / 256 * 256;
            }
            for (int c = 0; c < nco; c++) {
                ob[b].push_back(q);
                q += ((size_t)ocap * type_width(on.types[c]) + 255) / 256 * 256;
            }
            nd[b] = (int64_t *)q;
        }
        std::vector<rw_relation_in> din(in, in + nin);   // other inputs are unused by this plan
        int64_t total = 0;
        auto drain = [&](int64_t k) {      // compacted rows of chunk k -> host, appended
            const int b = (int)(k & 1);
            cuda_check(cudaEventSynchronize(ev_cnt[b]), "sync count");
            const int64_t nk = hcnt[b];
            const int64_t rows = std::max<int64_t>(0, std::min(nk, out->capacity - total));
            for (int c = 0; c < nco; c++)
                if (rows > 0)
                    cuda_check(cudaMemcpyAsync((char *)out->cols[c] + (size_t)total * type_width(on.types[c]), ob[b][c],
                                               (size_t)rows * type_width(on.types[c]), cudaMemcpyDeviceToHost, sd),
                               "D2H");
            cuda_check(cudaEventRecord(ev_out_free[b], sd), "event");
            total += nk;
        };
        int64_t launches = 0;
        for (int64_t k = 0; k < nch; k++) {
            const int b = (int)(k & 1);
            const int64_t r0 = k * C, rows = std::min(C, ri.n - r0);
            if (k >= 2)
                cuda_check(cudaStreamWaitEvent(sh, ev_in_free[b], 0), "wait");
            for (int c = 0; c < nci; c++)
                cuda_check(cudaMemcpyAsync(ib[b][c], (const char *)ri.cols[c] + (size_t)r0 * type_width(sn.types[c]),
                                           (size_t)rows * type_width(sn.types[c]), cudaMemcpyHostToDevice, sh),
                           "H2D");
            cuda_check(cudaEventRecord(ev_h2d[b], sh), "event");
            cuda_check(cudaStreamWaitEvent(p->stream, ev_h2d[b], 0), "wait");
            if (k >= 2 && !agg)
                cuda_check(cudaStreamWaitEvent(p->stream, ev_out_free[b], 0), "wait");
            std::vector<const void *> cc(ib[b].begin(), ib[b].end());
            din[sn.input_index].n = rows;
            din[sn.input_index].cols = cc.data();
            rw_relation_out dout{ob[b].data(), ocap, nd[b], -1};
            p->defer_finalize = agg && k + 1 < nch;
            execute(p, din.data(), nin, out_node, &dout);
            launches += p->launches;
            cuda_check(cudaEventRecord(ev_in_free[b], p->stream), "event");
            cuda_check(cudaMemcpyAsync(hcnt + b, nd[b], 8, cudaMemcpyDeviceToHost, p->stream), "copy count");
            cuda_check(cudaEventRecord(ev_cnt[b], p->stream), "event");
            if (!agg && k >= 1)
                drain(k - 1);
        }
        drain(nch - 1);
        cuda_check(cudaStreamSynchronize(sd), "sync");
        cuda_check(cudaStreamSynchronize(p->stream), "sync");
        if (agg) {
            cuda_check(cudaMemcpy(p->jtot_host + 8, p->err, 16, cudaMemcpyDeviceToHost), "copy err");
            raise_agg_errors(p);
        }
        out->n = total;
        p->launches = launches;
    } catch (...) {
        cleanup();
        throw;
    }
    cleanup();
    if (out->n > out->capacity)
        raise(RW_E_CAPACITY, "output needs " + std::to_string(out->n) + " rows, capacity " +
                                 std::to_string(out->capacity));
    return true;
}

std::string explain(rw_plan *p, int out_node)
{
    node_at(p, out_node);
    std::ostringstream s;
    static const char *kn[] = {"INPUT", "SELECT", "PROJECT", "JOIN", "AGG", "SETOP"};
    Grouping G = build_groups(p, out_node);
    s << "plan: " << p->nodes.size() << " nodes, output node " << out_node << ", fuse=" << p->o.fuse << "\n";
    s << "edges:\n";
    for (size_t i = 0; i < p->nodes.size(); i++) {
        if (!G.reach[i]) continue;
        const Node &n = p->nodes[i];
        for (int pr : {n.in, n.left, n.right}) {
            if (pr < 0) continue;
            int gp = p->nodes[pr].kind == N_INPUT ? -1 : G.produced_by.count(pr) ? G.produced_by[pr] : -2;
            int gc = -3;
            for (size_t q = 0; q < G.groups.size(); q++) {
                const Group &g = G.groups[q];
                if (g.out == (int)i || g.join == (int)i || g.join_in == (int)i || g.agg == (int)i ||
                    std::find(g.chain.begin(), g.chain.end(), (int)i) != g.chain.end() ||
                    std::find(g.pre.begin(), g.pre.end(), (int)i) != g.pre.end() ||
                    std::find(g.prechain[0].begin(), g.prechain[0].end(), (int)i) != g.prechain[0].end() ||
                    std::find(g.prechain[1].begin(), g.prechain[1].end(), (int)i) != g.prechain[1].end() ||
                    std::find(g.prechain[2].begin(), g.prechain[2].end(), (int)i) != g.prechain[2].end())
                    gc = (int)q;
            }
            bool fused = false;
            if (gc >= 0) {
                const Group &g = G.groups[gc];
                fused = pr == g.join || (g.join_in >= 0 && pr == g.join_in) ||
                        std::find(g.chain.begin(), g.chain.end(), pr) != g.chain.end() ||
                        std::find(g.pre.begin(), g.pre.end(), pr) != g.pre.end() ||
                        std::find(g.prechain[0].begin(), g.prechain[0].end(), pr) != g.prechain[0].end() ||
                        std::find(g.prechain[1].begin(), g.prechain[1].end(), pr) != g.prechain[1].end() ||
                        std::find(g.prechain[2].begin(), g.prechain[2].end(), pr) != g.prechain[2].end();
            }
            (void)gp;
            s << "  " << pr << "(" << kn[p->nodes[pr].kind] << ") -> " << i << "(" << kn[n.kind]
              << "): " << dep_name(classify_edge(p, pr, (int)i)) << " dependence, "
              << (fused ? "fused" : "materialised") << "\n";
        }
    }
    for (int c : G.cuts)
        s << "split by the resource budget (Algorithm 2, P:167-171): node " << c << "(" << kn[p->nodes[c].kind]
          << ") materialised\n";
    s << "groups:\n";
    for (size_t q = 0; q < G.groups.size(); q++) {
        const Group &g = G.groups[q];
        s << "  group " << q << ": "
          << (g.kind == G_SCAN ? "k_scan_chain"
                               : g.kind == G_SET ? "k_set_splits+k_set_op+k_set_scan+k_set_op<write>"
                                                 : (g.join_in >= 0 ? "k_jsplit+k_jmatch x2 (chained)+k_jtiles+k_join_emit<3-input>"
                                                                   : "k_jsplit+k_jmatch+k_jtiles+k_join_emit<2-input>"));
        if (g.agg >= 0) s << "<agg>+k_agg_finalize";
        s << " nodes [";
        if (g.kind == G_SCAN) s << "src " << g.source;
        else if (g.kind == G_SET) s << "setop " << g.join;
        else if (g.join_in >= 0) s << "joins " << g.join_in << " -> " << g.join << " (3 inputs, mixed-radix expansion)";
        else s << "join " << g.join;
        for (int c : g.pre) s << ", key SELECT " << c << " (fused into the run matching)";
        for (int sd = 0; sd < 3; sd++)
            for (int c : g.prechain[sd])
                s << ", " << kn[p->nodes[c].kind] << " " << c << " (upstream of the join, input " << sd
                  << ", fused into the expansion)";
        for (int c : g.chain) s << ", " << kn[p->nodes[c].kind] << " " << c;
        if (g.agg >= 0) s << ", AGG " << g.agg;
        s << "] -> node " << g.out;
        if (g.kind == G_SET) {
            s << " | merge-path partitions of " << set_partition_rows() << " merged rows, smem "
              << set_op_smem((int)p->nodes[g.join].types.size()) << " B\n";
            continue;
        }
        try {
            Lowered L;
            std::vector<int> st = g.kind == G_SCAN ? p->nodes[g.source].types : join_src_types(p, g);
            lower(p, g, st, L);
            if (L.emit)
                s << " | emitting kernel k_scan_emit<" << L.nt << "," << L.items << (L.teams > 1 ? ",2 teams" : "") << ">"
                  << (L.direct ? ", direct (no SELECT)" : "");
            s << " | tile " << L.tile << " rows (" << L.items << "/thread), stages " << L.stages << ", out ring " << L.out_bytes << " B"
              << ", smem " << L.smem
              << " B, CTAs/SM " << L.ctas << ", slots " << L.P.nslots << " (" << L.P.nin << " loaded), ops "
              << L.P.nops;
            if (L.agg)
            {
                s << ", groups " << L.P.D << ", sums " << L.P.nagg;
                if (L.P.agg_mode == 2)
                    s << ", register one-hot terminal" << (L.P.q1fused ? " (Q1 program fused per row)" : "");
                else if (L.P.agg_mode == 3)
                    s << ", global-atomic terminal";
                else
                    s << ", partial flush every " << L.P.flush_rows << " rows";
            }
        } catch (const RwError &e) {
            s << " | not lowerable: " << e.msg;
        }
        s << "\n";
    }
    return s.str();
}

}  // namespace

// ===========================================================================
// C ABI
// ===========================================================================
#define RW_TRY try {
#define RW_CATCH                                          \
    }                                                     \
    catch (const RwError &e)                              \
    {                                                     \
        g_err = e.msg;                                    \
        return e.s;                                       \
    }                                                     \
    catch (const std::bad_alloc &)                        \
    {                                                     \
        g_err = "host out of memory";                     \
        return RW_E_OOM;                                  \
    }                                                     \
    catch (...)                                           \
    {                                                     \
        g_err = "unexpected internal error";              \
        return RW_E_STATE;                                \
    }

extern "C" {

const char *rw_status_str(rw_status s)
{
    switch (s) {
    case RW_OK: return "RW_OK";
    case RW_E_ARG: return "RW_E_ARG";
    case RW_E_TYPE: return "RW_E_TYPE";
    case RW_E_UNSORTED: return "RW_E_UNSORTED";
    case RW_E_OVERFLOW: return "RW_E_OVERFLOW";
    case RW_E_UNSUPPORTED: return "RW_E_UNSUPPORTED";
    case RW_E_CAPACITY: return "RW_E_CAPACITY";
    case RW_E_OOM: return "RW_E_OOM";
    case RW_E_CUDA: return "RW_E_CUDA";
    case RW_E_DOMAIN: return "RW_E_DOMAIN";
    case RW_E_STATE: return "RW_E_STATE";
    }
    return "RW_E_?";
}

const char *rw_last_error(void) { return g_err.c_str(); }

rw_status rw_plan_create(rw_plan **out, const rw_plan_opts *opts)
{
    RW_TRY
    if (!out)
        raise(RW_E_ARG, "null out");
    rw_plan_opts o{};
    o.fuse = 1;
    if (opts)
        o = *opts;
    int ndev = 0;
    cuda_check(cudaGetDeviceCount(&ndev), "cudaGetDeviceCount");
    if (o.device < 0 || o.device >= ndev)
        raise(RW_E_ARG, "no such CUDA device");
    cuda_check(cudaSetDevice(o.device), "cudaSetDevice");
    int major = 0;
    cuda_check(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, o.device), "attr");
    if (major != 10)
        raise(RW_E_CUDA, "librw is built for sm_100a (B200) only");
    rw_plan *p = new rw_plan();
    p->o = o;
    p->stream = (cudaStream_t)o.cuda_stream;
    cuda_check(cudaDeviceGetAttribute(&p->sms, cudaDevAttrMultiProcessorCount, o.device), "attr");
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, o.device) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    try {
        p->ctrs = (uint32_t *)dev_alloc(p, 64);
        cuda_check(cudaMemsetAsync(p->ctrs, 0, 64, p->stream), "memset");
        p->jtot = (int64_t *)dev_alloc(p, 64);
        p->err = (int32_t *)dev_alloc(p, 64);
        cuda_check(cudaMemsetAsync(p->err, 0, 64, p->stream), "memset");
        cuda_check(cudaMallocHost(&p->jtot_host, 128), "cudaMallocHost");
        ensure_status(p, 4096);
        cuda_check(cudaStreamSynchronize(p->stream), "sync");
    } catch (...) {
        delete p;
        throw;
    }
    *out = p;
    return RW_OK;
    RW_CATCH
}

void rw_plan_destroy(rw_plan *p)
{
    if (!p)
        return;
    cudaSetDevice(p->o.device);
    cudaStreamSynchronize(p->stream);
    for (auto &kv : p->agg_acc)
        cudaFree(kv.second);
    if (p->status) cudaFree(p->status);
    if (p->ctrs) cudaFree(p->ctrs);
    if (p->cnt) cudaFree(p->cnt);
    if (p->jtot) cudaFree(p->jtot);
    if (p->err) cudaFree(p->err);
    if (p->gring) cudaFree(p->gring);
    if (p->jtot_host) cudaFreeHost(p->jtot_host);
    if (p->hs.init) {
        cudaStreamSynchronize(p->hs.sh);
        cudaStreamSynchronize(p->hs.sd);
        if (p->hs.buf) cudaFree(p->hs.buf);
        cudaFreeHost(p->hs.hcnt);
        for (int a = 0; a < 4; a++)
            for (int b = 0; b < 2; b++)
                cudaEventDestroy(p->hs.ev[a][b]);
        cudaStreamDestroy(p->hs.sh);
        cudaStreamDestroy(p->hs.sd);
    }
    delete p;
}

static int add_node(rw_plan *p, Node &&n, int32_t *node)
{
    p->nodes.push_back(std::move(n));
    int id = (int)p->nodes.size() - 1;
    if (node)
        *node = id;
    return id;
}

static void check_type(int t)
{
    if (t < RW_I32 || t > RW_U8)
        raise(RW_E_TYPE, "unknown attribute type " + std::to_string(t));
}

rw_status rw_plan_add_input(rw_plan *p, int32_t ncols, const int32_t *types, int32_t nkey_sorted,
                            const int64_t *lo, const int64_t *hi, int32_t *node)
{
    RW_TRY
    if (!p || ncols < 1 || ncols > kMaxOut || !types || nkey_sorted < 0 || nkey_sorted > ncols)
        raise(RW_E_ARG, "bad input declaration");
    Node n;
    n.kind = N_INPUT;
    for (int c = 0; c < ncols; c++) {
        check_type(types[c]);
        n.types.push_back(types[c]);
        Interval r = type_range(types[c]);
        if (lo) r.lo = std::max<i128>(r.lo, lo[c]);
        if (hi) r.hi = std::min<i128>(r.hi, types[c] == T_U64 ? (i128)(uint64_t)hi[c] : (i128)hi[c]);
        if (r.lo > r.hi)
            raise(RW_E_ARG, "empty bound interval for column " + std::to_string(c));
        n.bounds.push_back(r);
    }
    n.nkey_sorted = nkey_sorted;
    n.input_index = (int)p->inputs.size();
    int id = add_node(p, std::move(n), node);
    p->inputs.push_back(id);
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_add_select(rw_plan *p, int32_t in, const rw_pred *pr, int32_t np, int32_t *node)
{
    RW_TRY
    if (!p || np < 0 || (np > 0 && !pr))
        raise(RW_E_ARG, "bad select");
    const Node &src = node_at(p, in);
    Node n;
    n.kind = N_SELECT;
    n.in = in;
    n.types = src.types;
    n.bounds = src.bounds;
    n.nkey_sorted = src.nkey_sorted;
    const int nc = (int)src.types.size();
    for (int i = 0; i < np; i++) {
        const rw_pred &a = pr[i];
        if (a.col < 0 || a.col >= nc || a.op < RW_LT || a.op > RW_NE)
            raise(RW_E_ARG, "bad select atom " + std::to_string(i));
        if (a.rhs_is_col) {
            if (a.rhs_col < 0 || a.rhs_col >= nc)
                raise(RW_E_ARG, "bad select atom rhs column");
            if (src.types[a.rhs_col] != src.types[a.col])
                raise(RW_E_TYPE, "column-vs-column atom needs identical types");
        }
        n.preds.push_back(a);
    }
    add_node(p, std::move(n), node);
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_add_project(rw_plan *p, int32_t in, const rw_expr *e, int32_t ne, const int32_t *roots,
                              int32_t nout, int32_t *node)
{
    RW_TRY
    if (!p || ne < 1 || !e || !roots || nout < 1 || nout > kMaxOut)
        raise(RW_E_ARG, "bad project");
    const Node &src = node_at(p, in);
    const int nc = (int)src.types.size();
    for (int i = 0; i < ne; i++) {
        const rw_expr &x = e[i];
        if (x.op < RW_COL || x.op > RW_DIVC)
            raise(RW_E_ARG, "bad expression op");
        check_type(x.type);
        if (x.type == RW_U8 && x.op != RW_COL)
            raise(RW_E_TYPE, "u8 results only for column references");
        if (x.op == RW_COL && (x.a < 0 || x.a >= nc))
            raise(RW_E_ARG, "expression column out of range");
        if ((x.op == RW_ADD || x.op == RW_SUB || x.op == RW_MUL) &&
            (x.a < 0 || x.a >= i || x.b < 0 || x.b >= i))
            raise(RW_E_ARG, "expression operands must be earlier nodes");
        if (x.op == RW_DIVC) {
            if (x.a < 0 || x.a >= i)
                raise(RW_E_ARG, "expression operands must be earlier nodes");
            if (wrap_to(x.type, x.k) == 0)
                raise(RW_E_ARG, "division by zero constant");
        }
    }
    Node n;
    n.kind = N_PROJECT;
    n.in = in;
    n.exprs.assign(e, e + ne);
    std::vector<Interval> memo(ne);
    std::vector<char> done(ne, 0);
    for (int j = 0; j < nout; j++) {
        if (roots[j] < 0 || roots[j] >= ne)
            raise(RW_E_ARG, "bad root");
        n.roots.push_back(roots[j]);
        n.types.push_back(e[roots[j]].type);
        n.bounds.push_back(expr_interval(src, n.exprs, roots[j], memo, done, p->o.strict_overflow != 0));
    }
    // key-preserving prefix: leading outputs that are plain references to the
    // input's leading sorted columns, in order, with unchanged type
    int k = 0;
    while (k < nout && k < src.nkey_sorted) {
        const rw_expr &x = e[roots[k]];
        if (x.op != RW_COL || x.a != k || x.type != src.types[k]) break;
        k++;
    }
    n.nkey_sorted = k;
    add_node(p, std::move(n), node);
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_add_join(rw_plan *p, int32_t left, int32_t right, int32_t nkey, int32_t *node)
{
    RW_TRY
    if (!p)
        raise(RW_E_ARG, "null plan");
    const Node &L = node_at(p, left);
    const Node &R = node_at(p, right);
    if (nkey < 1 || nkey > (int)L.types.size() || nkey > (int)R.types.size())
        raise(RW_E_ARG, "bad nkey");
    for (int c = 0; c < nkey; c++)
        if (L.types[c] != R.types[c])
            raise(RW_E_TYPE, "join key types differ");
    // keys are matched on one order-preserving image of at most 8 bytes: one column of
    // any type, or two columns of at most 4 bytes each (lexicographic, A7)
    if (nkey > 2 || (nkey == 2 && (type_width(L.types[0]) == 8 || type_width(L.types[1]) == 8)))
        raise(RW_E_UNSUPPORTED, "join keys: one column, or two columns of at most 4 bytes each");
    if (L.nkey_sorted < nkey || R.nkey_sorted < nkey)
        raise(RW_E_UNSORTED, "join inputs must be sorted on the key (kernel dependence: sort first)");
    if (L.kind == N_AGG || R.kind == N_AGG)
        ;  // AGG output is sorted by group code: legal, materialised (kernel dependence)
    Node n;
    n.kind = N_JOIN;
    n.left = left;
    n.right = right;
    n.nkey = nkey;
    for (size_t c = 0; c < L.types.size(); c++) {
        n.types.push_back(L.types[c]);
        Interval b = L.bounds[c];
        if (c < (size_t)nkey) {
            b.lo = std::max(b.lo, R.bounds[c].lo);
            b.hi = std::min(b.hi, R.bounds[c].hi);
            if (b.lo > b.hi) b = L.bounds[c];
        }
        n.bounds.push_back(b);
    }
    for (size_t c = nkey; c < R.types.size(); c++) {
        n.types.push_back(R.types[c]);
        n.bounds.push_back(R.bounds[c]);
    }
    if ((int)n.types.size() > kMaxOut)
        raise(RW_E_UNSUPPORTED, "join output wider than 32 columns");
    n.nkey_sorted = nkey;
    add_node(p, std::move(n), node);
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_add_setop(rw_plan *p, int32_t left, int32_t right, int32_t op, int32_t *node)
{
    RW_TRY
    if (!p)
        raise(RW_E_ARG, "null plan");
    const Node &L = node_at(p, left);
    const Node &R = node_at(p, right);
    if (op != RW_UNION && op != RW_INTERSECT && op != RW_DIFFERENCE)
        raise(RW_E_ARG, "bad set operator");
    if (L.types != R.types)
        raise(RW_E_TYPE, "set operator inputs need identical schemas");
    if ((int)L.types.size() > kMaxSetCols)
        raise(RW_E_UNSUPPORTED, "set operators take at most 4 columns");
    if (L.nkey_sorted < (int)L.types.size() || R.nkey_sorted < (int)R.types.size())
        raise(RW_E_UNSORTED, "set operator inputs must be sorted on every column");
    Node n;
    n.kind = N_SETOP;
    n.left = left;
    n.right = right;
    n.setop = op;
    n.types = L.types;
    for (size_t c = 0; c < L.types.size(); c++) {
        Interval b = L.bounds[c];
        if (op == RW_UNION) {
            b.lo = std::min(b.lo, R.bounds[c].lo);
            b.hi = std::max(b.hi, R.bounds[c].hi);
        }
        n.bounds.push_back(b);
    }
    n.nkey_sorted = (int)n.types.size();
    add_node(p, std::move(n), node);
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_add_agg(rw_plan *p, int32_t in, const int32_t *gcols, const int32_t *gdomain, int32_t ng,
                          const rw_agg *a, int32_t na, int32_t *node)
{
    RW_TRY
    if (!p || ng < 0 || ng > kMaxGroupCols || na < 0 || na > kMaxAggs || (ng && (!gcols || !gdomain)) ||
        (na && !a))
        raise(RW_E_ARG, "bad agg");
    const Node &src = node_at(p, in);
    const int nc = (int)src.types.size();
    Node n;
    n.kind = N_AGG;
    n.in = in;
    int64_t D = 1;
    int nsum = 0, ncols = ng;
    for (int c = 0; c < ng; c++) {
        if (gcols[c] < 0 || gcols[c] >= nc || gdomain[c] < 1)
            raise(RW_E_ARG, "bad group column");
        D *= gdomain[c];
        if (D > kMaxAggSlots)
            raise(RW_E_UNSUPPORTED, "group domain product above 4096");
        n.gcols.push_back(gcols[c]);
        n.gdomain.push_back(gdomain[c]);
        n.types.push_back(src.types[gcols[c]]);
        n.bounds.push_back({0, gdomain[c] - 1});
    }
    for (int q = 0; q < na; q++) {
        if (a[q].op == RW_SUM) {
            if (a[q].col < 0 || a[q].col >= nc)
                raise(RW_E_ARG, "bad aggregate column");
            nsum++;
            n.types.push_back(RW_U64);
            n.bounds.push_back(type_range(T_U64));
            n.types.push_back(RW_I64);
            n.bounds.push_back(type_range(T_I64));
            ncols += 2;
        } else if (a[q].op == RW_COUNT) {
            n.types.push_back(RW_I64);
            n.bounds.push_back({0, INT64_MAX});
            ncols += 1;
        } else {
            raise(RW_E_ARG, "bad aggregate op");
        }
        n.aggs.push_back(a[q]);
    }
    if (ncols > kMaxOut || D * (nsum + 1) > kMaxAggSlots)
        raise(RW_E_UNSUPPORTED, "aggregate too wide");
    n.D = (int)D;
    n.nkey_sorted = ng;
    add_node(p, std::move(n), node);
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_node_schema(const rw_plan *p, int32_t node, int32_t *ncols, int32_t *types)
{
    RW_TRY
    if (!p || !ncols)
        raise(RW_E_ARG, "null argument");
    const Node &n = node_at(p, node);
    *ncols = (int32_t)n.types.size();
    if (types)
        for (size_t c = 0; c < n.types.size(); c++)
            types[c] = n.types[c];
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_execute(rw_plan *p, const rw_relation_in *in, int32_t nin, int32_t out_node,
                          rw_relation_out *out)
{
    RW_TRY
    if (!p)
        raise(RW_E_ARG, "null plan");
    execute(p, in, nin, out_node, out);
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_execute_multi(rw_plan *p, const rw_relation_in *in, int32_t nin, const int32_t *out_nodes,
                                int32_t nout, rw_relation_out *outs)
{
    RW_TRY
    if (!p)
        raise(RW_E_ARG, "null plan");
    execute_multi(p, in, nin, out_nodes, nout, outs);
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_execute_host(rw_plan *p, const rw_relation_in *in, int32_t nin, int32_t out_node,
                               rw_relation_out *out)
{
    RW_TRY
    if (!p || !out)
        raise(RW_E_ARG, "null argument");
    check_inputs(p, in, nin);
    cuda_check(cudaSetDevice(p->o.device), "cudaSetDevice");
    if (execute_host_streamed(p, in, nin, out_node, out))
        return RW_OK;
    std::vector<void *> dev;
    std::vector<std::vector<const void *>> dcols(nin);
    std::vector<rw_relation_in> din(nin);
    auto cleanup = [&]() {
        for (void *d : dev)
            cudaFreeAsync(d, p->stream);
    };
    try {
        for (int i = 0; i < nin; i++) {
            const Node &n = p->nodes[p->inputs[i]];
            for (size_t c = 0; c < n.types.size(); c++) {
                size_t bytes = (size_t)in[i].n * type_width(n.types[c]);
                void *d = dev_alloc(p, bytes);
                dev.push_back(d);
                if (bytes)
                    cuda_check(cudaMemcpyAsync(d, in[i].cols[c], bytes, cudaMemcpyHostToDevice, p->stream), "H2D");
                dcols[i].push_back(d);
            }
            din[i].n = in[i].n;
            din[i].cols = dcols[i].data();
        }
        const Node &on = node_at(p, out_node);
        std::vector<void *> ocols;
        for (int t : on.types) {
            void *d = dev_alloc(p, (size_t)std::max<int64_t>(out->capacity, 1) * type_width(t));
            dev.push_back(d);
            ocols.push_back(d);
        }
        rw_relation_out dout{ocols.data(), out->capacity, nullptr, -1};
        rw_status st = RW_OK;
        try {
            execute(p, din.data(), nin, out_node, &dout);
        } catch (const RwError &e) {
            if (e.s != RW_E_CAPACITY)
                throw;
            st = e.s;
            g_err = e.msg;
        }
        const int64_t rows = std::min(dout.n, out->capacity);
        for (size_t c = 0; c < on.types.size(); c++)
            if (rows > 0)
                cuda_check(cudaMemcpyAsync(out->cols[c], ocols[c], (size_t)rows * type_width(on.types[c]),
                                           cudaMemcpyDeviceToHost, p->stream),
                           "D2H");
        cleanup();
        cuda_check(cudaStreamSynchronize(p->stream), "sync");
        out->n = dout.n;
        return st;
    } catch (...) {
        cleanup();
        throw;
    }
    RW_CATCH
}

rw_status rw_plan_explain(rw_plan *p, int32_t out_node, char *buf, size_t cap)
{
    RW_TRY
    if (!p || !buf || cap == 0)
        raise(RW_E_ARG, "bad buffer");
    cuda_check(cudaSetDevice(p->o.device), "cudaSetDevice");
    std::string s = explain(p, out_node);
    size_t n = std::min(cap - 1, s.size());
    std::memcpy(buf, s.data(), n);
    buf[n] = 0;
    return s.size() < cap ? RW_OK : RW_E_CAPACITY;
    RW_CATCH
}

int64_t rw_plan_last_launches(const rw_plan *p) { return p ? p->launches : -1; }

rw_status rw_split_by_splitters(const void *keys_dev, int64_t n, int32_t key_type, const void *splitters_dev,
                                int32_t nsplit, int64_t *bounds_dev, void *cuda_stream)
{
    RW_TRY
    if (n < 0 || nsplit < 0 || (n > 0 && !keys_dev) || (nsplit > 0 && (!splitters_dev || !bounds_dev)))
        raise(RW_E_ARG, "bad split arguments");
    check_type(key_type);
    cuda_check(split_bounds_launch(keys_dev, n, key_type, splitters_dev, nsplit, bounds_dev,
                                   (cudaStream_t)cuda_stream),
               "k_split_bounds");
    return RW_OK;
    RW_CATCH
}

// Single-pass P-way merge (merge_p.cu) of runs whose tuples pack into <= 8 bytes.
// `packed` (u64 tuple images) or `cols` is the input; temporaries from cudaMallocAsync.
static void merge_runs_single_pass(const void *const *cols, const uint64_t *packed, const int32_t *types,
                                   int32_t ncols, const int64_t *run_off, int32_t nrun, void *const *out_cols,
                                   cudaStream_t st)
{
    MpLaunch M{};
    for (int c = 0; c < ncols; c++) {
        M.col[c] = cols ? cols[c] : nullptr;
        M.types[c] = (uint8_t)types[c];
        M.out[c] = out_cols[c];
    }
    M.ncols = ncols;
    M.packed = packed;
    M.nrun = nrun;
    M.G = nrun;
    M.T = std::max(1, kMpC / (M.G + nrun));   // a group holds <= (G + P) * T <= kMpC elements
    M.samp_base[0] = 0;
    for (int q = 0; q <= nrun; q++) {
        M.run_off[q] = run_off[q];
        if (q < nrun) {
            const int64_t nq = run_off[q + 1] - run_off[q];
            if (nq >= (int64_t)UINT32_MAX)
                raise(RW_E_UNSUPPORTED, "merge run of 2^32 rows or more");
            M.samp_base[q + 1] = M.samp_base[q] + (nq + M.T - 1) / M.T;
        }
    }
    M.S = M.samp_base[nrun];
    M.NG = (M.S + M.G - 1) / M.G;
    if (M.S == 0)
        return;
    int dev = 0, sms = 148;
    cuda_check(cudaGetDevice(&dev), "cudaGetDevice");
    cuda_check(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev), "attr");
    void *sv = nullptr, *cuts = nullptr, *bound = nullptr;
    cuda_check(cudaMallocAsync(&sv, (size_t)M.S * 8, st), "cudaMallocAsync");
    cudaError_t e1 = cudaMallocAsync(&cuts, (size_t)M.NG * nrun * 4, st);
    cudaError_t e2 = cudaMallocAsync(&bound, (size_t)M.NG * 8, st);
    cudaError_t e3 = cudaSuccess;
    if (e1 == cudaSuccess && e2 == cudaSuccess) {
        M.sv = (uint64_t *)sv;
        M.cuts = (uint32_t *)cuts;
        M.bound = (int64_t *)bound;
        e3 = mp_merge_launch(M, sms, st);
    }
    cudaFreeAsync(sv, st);
    if (cuts)
        cudaFreeAsync(cuts, st);
    if (bound)
        cudaFreeAsync(bound, st);
    cuda_check(e1, "cudaMallocAsync");
    cuda_check(e2, "cudaMallocAsync");
    cuda_check(e3, "k_mp_merge");
}

static bool packable(const int32_t *types, int32_t ncols)
{
    int bytes = 0;
    for (int c = 0; c < ncols; c++)
        bytes += type_width(types[c]);
    return bytes <= 8;
}

rw_status rw_merge_runs(const void *const *cols, const int32_t *types, int32_t ncols, const int64_t *run_off,
                        int32_t nrun, void *const *out_cols, void *cuda_stream)
{
    RW_TRY
    if (ncols < 1 || ncols > kMaxMergeCols || nrun < 0 || !cols || !types || !run_off || !out_cols)
        raise(RW_E_ARG, "bad merge arguments");
    cudaStream_t st = (cudaStream_t)cuda_stream;
    MergeTypes T{};
    for (int c = 0; c < ncols; c++) {
        check_type(types[c]);
        T.t[c] = (uint8_t)types[c];
    }
    for (int r = 0; r < nrun; r++)
        if (run_off[r + 1] < run_off[r])
            raise(RW_E_ARG, "run offsets must be non-decreasing");
    if (nrun >= 2 && nrun <= kMpMaxRuns && packable(types, ncols)) {
        // one read and one write of the data (merge_p.cu)
        std::vector<int64_t> off(run_off, run_off + nrun + 1);
        for (auto &o : off)
            o -= run_off[0];
        std::vector<const void *> base(ncols);
        for (int c = 0; c < ncols; c++)
            base[c] = (const char *)cols[c] + (size_t)run_off[0] * type_width(types[c]);
        merge_runs_single_pass(base.data(), nullptr, types, ncols, off.data(), nrun, out_cols, st);
        return RW_OK;
    }
    struct Run {
        MergeCols c;
        int64_t n;
        bool temp;
    };
    std::vector<Run> runs;
    for (int r = 0; r < nrun; r++) {
        Run x{};
        x.n = run_off[r + 1] - run_off[r];
        for (int c = 0; c < ncols; c++)
            x.c.col[c] = (const char *)cols[c] + (size_t)run_off[r] * type_width(types[c]);
        runs.push_back(x);
    }
    const int64_t total = nrun ? run_off[nrun] - run_off[0] : 0;
    std::vector<void *> temps;
    auto release = [&]() {
        for (void *t : temps)
            cudaFreeAsync(t, st);
    };
    try {
        if (runs.size() <= 1) {
            for (int c = 0; c < ncols && total > 0; c++)
                cuda_check(cudaMemcpyAsync(out_cols[c], runs[0].c.col[c], (size_t)total * type_width(types[c]),
                                           cudaMemcpyDeviceToDevice, st),
                           "copy run");
        }
        // wide tuples / more than kMpMaxRuns runs: pairwise merge tree; the last round
        // writes the caller's columns
        while (runs.size() > 1) {
            std::vector<Run> next;
            const bool last = runs.size() == 2;
            for (size_t r = 0; r + 1 < runs.size(); r += 2) {
                Run m{};
                m.n = runs[r].n + runs[r + 1].n;
                MergeOut O{};
                for (int c = 0; c < ncols; c++) {
                    if (last) {
                        O.col[c] = out_cols[c];
                    } else {
                        void *p = nullptr;
                        cuda_check(cudaMallocAsync(&p, (size_t)std::max<int64_t>(m.n, 1) * type_width(types[c]), st),
                                   "cudaMallocAsync");
                        temps.push_back(p);
                        O.col[c] = p;
                    }
                    m.c.col[c] = O.col[c];
                }
                cuda_check(merge2_launch(runs[r].c, runs[r].n, runs[r + 1].c, runs[r + 1].n, O, ncols, T, st),
                           "k_merge2");
                next.push_back(m);
            }
            if (runs.size() % 2)
                next.push_back(runs.back());
            runs.swap(next);
        }
    } catch (...) {
        release();
        throw;
    }
    release();
    return RW_OK;
    RW_CATCH
}

rw_status rw_pack_tuples(const void *const *cols, const int32_t *types, int32_t ncols, int64_t n,
                         uint64_t *packed_dev, void *cuda_stream)
{
    RW_TRY
    if (ncols < 1 || ncols > kMaxMergeCols || n < 0 || !cols || !types || (n > 0 && !packed_dev))
        raise(RW_E_ARG, "bad pack arguments");
    for (int c = 0; c < ncols; c++)
        check_type(types[c]);
    if (!packable(types, ncols))
        raise(RW_E_UNSUPPORTED, "tuple wider than 8 bytes");
    MpLaunch M{};
    for (int c = 0; c < ncols; c++) {
        M.col[c] = cols[c];
        M.types[c] = (uint8_t)types[c];
    }
    M.ncols = ncols;
    int dev = 0, sms = 148;
    cuda_check(cudaGetDevice(&dev), "cudaGetDevice");
    cuda_check(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev), "attr");
    cuda_check(mp_pack_launch(M, n, packed_dev, sms, (cudaStream_t)cuda_stream), "k_mp_pack");
    return RW_OK;
    RW_CATCH
}

rw_status rw_merge_packed_runs(const uint64_t *packed_dev, const int32_t *types, int32_t ncols,
                               const int64_t *run_off, int32_t nrun, void *const *out_cols, void *cuda_stream)
{
    RW_TRY
    if (ncols < 1 || ncols > kMaxMergeCols || nrun < 0 || nrun > kMpMaxRuns || !types || !run_off || !out_cols)
        raise(RW_E_ARG, "bad merge arguments");
    for (int c = 0; c < ncols; c++)
        check_type(types[c]);
    if (!packable(types, ncols))
        raise(RW_E_UNSUPPORTED, "tuple wider than 8 bytes");
    for (int r = 0; r < nrun; r++)
        if (run_off[r + 1] < run_off[r])
            raise(RW_E_ARG, "run offsets must be non-decreasing");
    if (nrun == 0 || run_off[nrun] == run_off[0])
        return RW_OK;
    if (!packed_dev)
        raise(RW_E_ARG, "bad merge arguments");
    // nrun == 1 is a merge of one run: the same kernels unpack it
    std::vector<int64_t> off(run_off, run_off + nrun + 1);
    for (auto &o : off)
        o -= run_off[0];
    merge_runs_single_pass(nullptr, packed_dev + run_off[0], types, ncols, off.data(), nrun, out_cols,
                           (cudaStream_t)cuda_stream);
    return RW_OK;
    RW_CATCH
}

static AggXfer agg_xfer(const rw_plan *p, int32_t agg_node)
{
    const Node &a = node_at(p, agg_node);
    if (a.kind != N_AGG)
        raise(RW_E_ARG, "node is not an aggregate");
    AggXfer X{};
    X.ngc = (int)a.gcols.size();
    for (int c = 0; c < X.ngc; c++) {
        X.gdomain[c] = a.gdomain[c];
        X.gtype[c] = (uint8_t)a.types[c];
    }
    X.nreq = (int)a.aggs.size();
    int L = 1;
    for (int q = 0; q < X.nreq; q++) {
        X.is_sum[q] = a.aggs[q].op == RW_SUM;
        L += X.is_sum[q] ? 4 : 1;
    }
    X.D = a.D;
    X.L = L;
    return X;
}

rw_status rw_plan_agg_limbs(const rw_plan *p, int32_t agg_node, int64_t *nlimbs)
{
    RW_TRY
    if (!p || !nlimbs)
        raise(RW_E_ARG, "null argument");
    AggXfer X = agg_xfer(p, agg_node);
    *nlimbs = (int64_t)X.D * X.L;
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_agg_export(rw_plan *p, int32_t agg_node, const void *const *cols, const int64_t *n_dev,
                             int64_t n_host, int64_t *limbs_dev)
{
    RW_TRY
    if (!p || !cols || !limbs_dev)
        raise(RW_E_ARG, "null argument");
    AggXfer X = agg_xfer(p, agg_node);
    const int ncols = (int)p->nodes[agg_node].types.size();
    for (int c = 0; c < ncols; c++)
        X.col[c] = cols[c];
    cuda_check(cudaSetDevice(p->o.device), "cudaSetDevice");
    cuda_check(cudaMemsetAsync(limbs_dev, 0, (size_t)X.D * X.L * 8, p->stream), "memset limbs");
    cuda_check(agg_export_launch(X, n_dev, n_host, limbs_dev, p->stream), "k_agg_export");
    return RW_OK;
    RW_CATCH
}

rw_status rw_plan_agg_import(rw_plan *p, int32_t agg_node, const int64_t *limbs_dev, rw_relation_out *out)
{
    RW_TRY
    if (!p || !limbs_dev || !out || !out->cols)
        raise(RW_E_ARG, "null argument");
    AggXfer X = agg_xfer(p, agg_node);
    const int ncols = (int)p->nodes[agg_node].types.size();
    OutPtrs O{};
    for (int c = 0; c < ncols; c++)
        O.col[c] = out->cols[c];
    cuda_check(cudaSetDevice(p->o.device), "cudaSetDevice");
    int64_t *nd = out->n_dev ? out->n_dev : p->cnt;
    if (!nd) {
        p->cnt_cap = 8;
        p->cnt = (int64_t *)dev_alloc(p, 64);
        nd = p->cnt;
    }
    cuda_check(agg_import_launch(X, limbs_dev, O, out->capacity, nd, p->stream), "k_agg_import");
    out->n = -1;
    if (!out->n_dev) {
        cuda_check(cudaMemcpyAsync(p->jtot_host + 2, nd, 8, cudaMemcpyDeviceToHost, p->stream), "copy n");
        cuda_check(cudaStreamSynchronize(p->stream), "sync");
        out->n = p->jtot_host[2];
        if (out->n > out->capacity)
            raise(RW_E_CAPACITY, "aggregate output needs " + std::to_string(out->n) + " rows");
    }
    return RW_OK;
    RW_CATCH
}

}  // extern "C"
