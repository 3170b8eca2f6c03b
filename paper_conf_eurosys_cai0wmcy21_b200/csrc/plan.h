// plan.h — host-only planning and lowering structures (no CUDA dependency).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "internal.h"

namespace dgcl {

// Topology D(V', E') of §5.1: a link i->j is a list of
// physical hops, hop h costs w[h] ticks per row.
struct Topology {
  int m = 0;
  std::vector<int64_t> w;          // ticks per row, per hop
  std::vector<int64_t> link_ptr;   // CSR over i*m + j
  std::vector<int32_t> link_hops;
  bool has(int i, int j) const { return link_ptr[i * m + j + 1] > link_ptr[i * m + j]; }
  static Topology uniform_nvswitch(int m);
};

// Communication relation: for every vertex u, the GPUs D_u that request
// it (ascending) and u's halo row pos_d(u) on each of them.
struct Relation {
  int64_t n = 0;
  int m = 0;
  std::vector<int64_t> d_ptr;  // [n+1]
  std::vector<int8_t> d_gpu;   // [S]
  std::vector<int32_t> d_pos;  // [S]
  std::vector<int64_t> n_halo; // [m] = |R_d|
};

// The plan S = union of trees T_u, edges grouped per vertex in planning order.
struct Plan {
  int m = 0;
  int n_stages = 0;                // max edge stage K
  std::vector<int64_t> order;      // planned vertices, in planning order
  std::vector<int64_t> e_ptr;      // [order.size()+1] edges of order[i]
  std::vector<int32_t> e_parent, e_child, e_stage;
  int64_t cost = 0;                // t(S) in ticks
  double seconds = 0;
  bool closed_form = false;        // planned by the uniform-switch closed form (parallel)
};

// Build the relation from the required lists; returns "" or an error message (EINVAL).
std::string build_relation(int64_t n, int m, const int32_t *part, const int64_t *req_ptr,
                           const int64_t *req_ids, Relation *out);

// SPST, Algorithm 1 + 2 (§5.2).  Returns "" or an error message (EPLAN).  allow_fast: on the
// uniform switch model use SPST's closed form (every tree a direct star; parallel), which gives
// the same plan as the general loop (tested)
std::string spst_plan(const Topology &topo, const int32_t *part, const Relation &rel,
                      uint64_t seed, Plan *out, bool allow_fast = true);

// A saved plan (trees, as dgcl_plan_export gives them) instead of SPST; the plan invariants are
// checked and t(S) recomputed.  Returns "" or an error message (EPLAN).
std::string import_plan(const Topology &topo, const int32_t *part, const Relation &rel,
                        int64_t n_edges, const int64_t *u, const int32_t *parent,
                        const int32_t *child, const int32_t *stage, Plan *out);

// ---- lowering ----------------------------------------------------------------------------

struct Lowered {
  int m = 0;
  int n_stages = 0;                      // forward stages K
  std::vector<DevGroup> groups;          // forward, backward, READY/WAIT, then direct-reduce
  int n_fwd_groups = 0;
  int direct_begin = 0, direct_end = 0;  // loopback direct-reduce backward groups (direct plans)
  int atomic_end = 0;  // [direct_end, atomic_end): loopback atomic-add backward groups (ablation)
  int fanout_end = 0;  // [atomic_end, fanout_end): forward stage-1 fan-out groups, one per owner
  int tree_end = 0;    // [fanout_end, tree_end): loopback tree-order backward (relay plans)
  // multicast (option "multicast"): [mc_begin, mc_end) = per-owner send groups (dst K_MCAST) and
  // per-(receiver, owner) unpack groups (src K_MCUC), inside the forward groups; the region holds
  // mc_total rows, owner s's at mc_off[s] ..
  int mc_begin = 0, mc_end = 0;
  std::vector<int64_t> mc_rows, mc_off;
  int64_t mc_total = 0;
  std::vector<int32_t> mc_unpack_wait;  // [d * m + s]: waits index of d's unpack of s, or -1
  std::vector<int32_t> idx;              // row index pool
  std::vector<int64_t> term_ptr;         // fold row pointers
  std::vector<uint32_t> terms;           // fold terms
  std::vector<DevWait> waits;
  // per-rank buffer rows
  std::vector<int64_t> n_halo, n_relay, n_slot;  // [m]
  int n_blocks = 1;  // vertex blocks of the stage chaining (relay plans), see ctr_index
  // relay plans, leaf split: forward deliveries no later stage forwards count on this block's
  // counters (nothing waits on them but the forward completion), -1 = no split
  int leaf_block = -1;
  // rows in: [dir][stage][block][src][dst] flattened
  std::vector<int64_t> rows_sd;
  int64_t &rows_at(int dir, int k, int s, int d, int b) {
    return rows_sd[(((size_t)(dir * kMaxStages + k) * kMaxBlocks + b) * m + s) * m + d];
  }
  int64_t rows(int dir, int k, int s, int d, int b) const {
    return rows_sd[(((size_t)(dir * kMaxStages + k) * kMaxBlocks + b) * m + s) * m + d];
  }
  int64_t rows(int dir, int k, int s, int d) const {  // all blocks
    int64_t t = 0;
    for (int b = 0; b < n_blocks; ++b) t += rows(dir, k, s, d, b);
    if (leaf_block >= n_blocks) t += rows(dir, k, s, d, leaf_block);
    return t;
  }
  int64_t n_relay_edges = 0;
  int64_t n_tree_edges = 0;
  double seconds = 0;
  int64_t table_bytes() const {
    return (int64_t)(idx.size() * 4 + term_ptr.size() * 8 + terms.size() * 4 +
                     waits.size() * sizeof(DevWait) + groups.size() * sizeof(DevGroup));
  }
};

// n_blocks: vertex blocks for the stage chaining of relay plans (1 = one counter per stage;
// single-stage plans always use 1); with_atomic / with_fanout: also build the ablation groups
// (atomic backward, fan-out forward) — only when their option is set (they cost lowering time)
// mc_min_fanout > 0: multicast the rows of vertices requested by >= that many GPUs
// (single-stage plans)
// leaf_split (relay plans, n_blocks = 1): 1 = deliveries of stages >= 2 that no later stage
// forwards get their own counters and come after the forwarded ones of their stage, 2 = stage 1
// too (by row: a row any of whose first hops forwards it counts as forwarded)
void lower_plan(const Relation &rel, const Plan &plan, const int32_t *part,
                const std::vector<int64_t> &loc, Lowered *out, int n_blocks = 1,
                bool with_atomic = false, bool with_fanout = false, int mc_min_fanout = 0,
                int leaf_split = 0);

// Work items for one launch: the groups `gids` (already in stage order, READY / WAIT groups
// included by the caller) cut into row ranges of about item_bytes gathered bytes and interleaved
// across the groups of a stage.  COPY items also get their row runs appended to `runs`
// (item.tp = first run, program-relative); items of short runs are flagged for gather4 (or for
// consumer gathers when direct_copy_rows > 0).  With `sterms`, FOLD groups whose rows fit are
// cut into STAGED items: every operand row (the destination rows a fold starts from, then each
// term's source row) is bulk-copied into the stage as segments of consecutive rows (appended to
// `runs`), and `sterms` receives each term's operand row (item.t0 = first, program-relative).
// The item limits follow the launch geometry (internal.h, TmaGeometry): operand bytes of one
// stage and rows per item (one meta slot of runs).
struct ItemLimits {
  int64_t operand_bytes;  // gathered bytes of one item (<= stage_bytes - kStageHdrBytes)
  int64_t max_rows;       // rows (COPY) / operand rows (staged FOLD) of one item
  int64_t min_items;      // COPY items per stage to aim for (co-resident CTAs; 0 = no spreading)
  bool align_sources = true;  // forward COPY groups of one source rank cut at common source rows
  bool lsu_gather = false;    // short-run COPY items gathered by the consumers (kItemLsu)
  int owner_major = 0;        // forward COPY items: 1 one executing rank's groups at a time,
                              // 2 one group at a time
};
ItemLimits item_limits(const TmaGeometry &g, int64_t item_bytes, int64_t min_items = 0);
void build_items(const Lowered &low, const std::vector<int32_t> &gids, int64_t row_bytes,
                 const ItemLimits &lim, bool signal_all, const std::vector<uint8_t> &needed_ctr,
                 std::vector<DevItem> *items, std::vector<DevRun> *runs,
                 int64_t direct_copy_rows = 0, std::vector<uint32_t> *sterms = nullptr);

// Relay forwards with the leaf split: reorder a launch's items so the forwarded rows of every
// stage run ahead of the leaves, with about lead_bytes of leaves between consecutive stages'
// forwarded items (< 0: keep the build order)
void lead_relay_items(const Lowered &low, std::vector<DevItem> *items, int64_t row_bytes,
                      int64_t lead_bytes);

}  // namespace dgcl
