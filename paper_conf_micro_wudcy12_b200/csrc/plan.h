// plan.h — host-side plan representation (DAG of RA operators), interval
// analysis, dependence classification and fusion grouping.  Internal.
#pragma once
#include <stdint.h>
#include <string>
#include <vector>
#include "../../include/rw.h"
#include "internal.h"

namespace rw {

typedef __int128 i128;

struct Interval {
    i128 lo, hi;
};

enum NodeKind { N_INPUT = 0, N_SELECT = 1, N_PROJECT = 2, N_JOIN = 3, N_AGG = 4, N_SETOP = 5 };

struct Node {
    NodeKind kind;
    std::vector<int> types;          // output schema
    std::vector<Interval> bounds;    // per output column value interval
    int nkey_sorted = 0;             // leading columns the output is sorted on
    int input_index = -1;            // N_INPUT: declaration order
    int in = -1, left = -1, right = -1;
    std::vector<rw_pred> preds;      // N_SELECT
    std::vector<rw_expr> exprs;      // N_PROJECT
    std::vector<int> roots;
    int nkey = 0;                    // N_JOIN
    int setop = 0;                   // N_SETOP: RW_UNION / RW_INTERSECT / RW_DIFFERENCE
    std::vector<int> gcols, gdomain; // N_AGG
    std::vector<rw_agg> aggs;
    int D = 1;
};

// Dependence class of a producer -> consumer edge (§4.1, Figure 8).
enum DepClass { DEP_THREAD = 0, DEP_CTA = 1, DEP_KERNEL = 2 };
const char *dep_name(int d);

// A fused group: one kernel template instance (plus its helper launches).
enum GroupKind { G_SCAN = 0, G_JOIN = 1, G_SET = 2 };
struct Group {
    GroupKind kind;
    int source = -1;                 // G_SCAN: producer node whose relation is scanned
    int join = -1;                   // G_JOIN: the JOIN node; G_SET: the set-operator node
    std::vector<int> chain;          // SELECT / PROJECT nodes fused after the source / join
    // input-dependence fusion (§4.4, Fig. 14(d)): several chains over the same
    // G_SCAN source, one output each (chain unused when non-empty)
    std::vector<std::vector<int>> branches;
    int agg = -1;                    // AGG terminal (or -1: materialising terminal)
    int out = -1;                    // node whose relation this group produces
    std::vector<int> deps;           // groups that must run first
    // G_JOIN: SELECT nodes on the join key fused into the run matching (N2); the
    // join then reads their source relations (jl, jr) directly
    std::vector<int> pre;            // absorbed SELECT nodes
    int jl = -1, jr = -1;            // relations feeding the join (after absorption)
    // 3-input group (JOIN -> JOIN on the same key, Fig. 14(b)): join_in = the inner JOIN
    // (inputs jl, jr), `join` the outer one (inner output, jc)
    int join_in = -1, jc = -1;
    // per input (A, B, C): SELECT / key-preserving PROJECT nodes upstream of the JOIN fused
    // into the expansion (source-to-join order); jl / jr / jc are then their raw sources
    std::vector<int> prechain[3];
};

Interval type_range(int t);
bool fits(const Interval &v, int t);
i128 wrap_to(int t, i128 v);

}  // namespace rw
