// lowering.cpp — plan trees -> executor groups (host only, no CUDA).
//
// §6.1: the plan S is organised into tuples (d_i, d_j, k, T^s_ij, T^r_ij):
// per stage k and GPU pair, the vertex ids d_i sends to d_j.  Here a tuple becomes one or more
// GROUPS, split by where the rows live on the sender (its embeddings, its halo, or its relay
// staging) and on the receiver (halo, or relay staging when the receiver only forwards), with the
// vertex ids already translated into row numbers of those buffers.  The receiver-side unpack of
// the paper is fused away: the sender writes each row at its final position.
//
// Backward: "stages are executed in a reverse order, and T^s_ij and T^r_ij are
// switched".  Forward edge p->c at stage k becomes the backward push c->p at stage b = K - k + 1,
// carrying c's partial sum val_c(u) into a per-(child, vertex) SLOT row on p.  The owner then
// folds its slots into emb_grad in ascending child order (RED, stage K + 1).  This replaces the
// paper's |D|-1 sub-stages with the same guarantee — every row has exactly one
// writer, no atomics — and additionally fixes the summation order (R6).

#include <algorithm>
#include <parallel/algorithm>
#include <cstdio>
#include <cstdlib>
#include <functional>
#include <chrono>
#include <cstring>
#include <deque>
#include <map>
#include <tuple>

#include "plan.h"

namespace dgcl {

namespace {

struct Entry {
  uint64_t key;
  int64_t sort2;
  int64_t edge;   // plan edge index
  int64_t vidx;   // index into plan.order
};

inline uint64_t pack_key(int stage, int exec, int dst, int a, int b) {
  return ((uint64_t)stage << 24) | ((uint64_t)exec << 16) | ((uint64_t)dst << 8) |
         ((uint64_t)a << 4) | (uint64_t)b;
}
// group key ordered (stage + block, stage, block, exec, dst, a, b): with vertex blocks the
// (stage, block) runs come in wavefront order — stage k of block b right after stage k - 1 of
// block b + 1 — so the executor reaches stage k of the first blocks while the later blocks'
// stage k - 1 still runs (every dependency, stage k - 1 of the same block, comes earlier);
// without blocks this is plain stage order
inline uint64_t pack_key_b(int stage, int block, int exec, int dst, int a, int b) {
  return ((uint64_t)(stage + block) << 40) | ((uint64_t)stage << 32) | ((uint64_t)block << 24) |
         ((uint64_t)exec << 16) | ((uint64_t)dst << 8) | ((uint64_t)a << 4) | (uint64_t)b;
}
inline int key_stage(uint64_t k) { return (int)(k >> 32 & 0xFF); }
inline int key_block(uint64_t k) { return (int)(k >> 24 & 0xFF); }

// position of u on GPU d (its halo row), or -1 if d did not request u
inline int32_t halo_pos(const Relation &rel, int64_t u, int d) {
  for (int64_t q = rel.d_ptr[u]; q < rel.d_ptr[u + 1]; ++q)
    if (rel.d_gpu[q] == d) return rel.d_pos[q];
  return -1;
}

}  // namespace

void lower_plan(const Relation &rel, const Plan &plan, const int32_t *part,
                const std::vector<int64_t> &loc, Lowered *out, int n_blocks, bool with_atomic,
                bool with_fanout, int mc_min_fanout, int leaf_split) {
  auto t0 = std::chrono::steady_clock::now();
  // DGCL_TIMING=1: per-section wall times on stderr (planning at scale, NEXT-4)
  static const bool timing = std::getenv("DGCL_TIMING") != nullptr;
  auto tl = t0;
  auto lap = [&](const char *what) {
    if (!timing) return;
    const auto now = std::chrono::steady_clock::now();
    std::fprintf(stderr, "[dgcl lowering] %-24s %8.3f s\n", what,
                 std::chrono::duration<double>(now - tl).count());
    tl = now;
  };
  const int m = plan.m;
  const int K = plan.n_stages;
  Lowered &L = *out;
  L = Lowered();
  L.m = m;
  L.n_stages = K;
  L.n_halo = rel.n_halo;
  L.n_relay.assign(m, 0);
  L.n_slot.assign(m, 0);
  L.rows_sd.assign((size_t)2 * kMaxStages * kMaxBlocks * m * m, 0);
  const int64_t NE = (int64_t)plan.e_parent.size();
  L.n_tree_edges = NE;
  const int64_t NV = (int64_t)plan.order.size();

  // Vertex blocks (relay plans): stage k of block b only waits for stage k-1 of block b, so a
  // stage's tail overlaps the next stage's first blocks instead of the launch idling at every
  // stage boundary.  Blocks are ranges of vertex ids holding about equal numbers of tree edges
  // (halo rows are ordered by id within an owner, so a block keeps runs of consecutive rows).
  const int NB = K >= 2 ? std::max(1, std::min(n_blocks, kMaxBlocks)) : 1;
  L.n_blocks = NB;
  std::vector<uint8_t> blk_of;  // per planned vertex index
  {
    const int64_t N = (int64_t)loc.size();
    std::vector<int64_t> w(N, 0);
    for (int64_t vi = 0; vi < NV; ++vi) w[plan.order[vi]] = plan.e_ptr[vi + 1] - plan.e_ptr[vi];
    std::vector<uint8_t> bu(N, 0);
    int64_t acc = 0;
    for (int64_t u = 0; u < N; ++u) {
      bu[u] = (uint8_t)std::min<int64_t>(NB - 1, NE > 0 ? acc * NB / NE : 0);
      acc += w[u];
    }
    blk_of.resize(NV);
    for (int64_t vi = 0; vi < NV; ++vi) blk_of[vi] = bu[plan.order[vi]];
  }

  // edge -> vertex index
  std::vector<int64_t> e_vidx(NE);
  for (int64_t i = 0; i < NV; ++i)
    for (int64_t e = plan.e_ptr[i]; e < plan.e_ptr[i + 1]; ++e) e_vidx[e] = i;
  // is the child of edge e a requester (halo) or a pure relay?
  std::vector<int32_t> child_pos(NE);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < NE; ++e)
    child_pos[e] = halo_pos(rel, plan.order[e_vidx[e]], plan.e_child[e]);
  // edge into node x of the same tree (for relay sources / children lists)
  auto edge_into = [&](int64_t vi, int x) -> int64_t {
    for (int64_t e = plan.e_ptr[vi]; e < plan.e_ptr[vi + 1]; ++e)
      if (plan.e_child[e] == x) return e;
    return -1;
  };

  // children index, built once (parallel over vertices): the tree edges out of the child node of
  // every edge, and out of every tree's root, each list in ascending child id (the fixed
  // contribution order, R6)
  std::vector<int64_t> kid_eptr(NE + 1, 0), kid_rptr(NV + 1, 0), kid_elist, kid_rlist;
  {
#pragma omp parallel for schedule(static)
    for (int64_t vi = 0; vi < NV; ++vi) {
      const int root = part[plan.order[vi]];
      int64_t nr = 0;
      for (int64_t e = plan.e_ptr[vi]; e < plan.e_ptr[vi + 1]; ++e) {
        int64_t nk = 0;
        for (int64_t f = plan.e_ptr[vi]; f < plan.e_ptr[vi + 1]; ++f)
          nk += plan.e_parent[f] == plan.e_child[e];
        kid_eptr[e + 1] = nk;
        nr += plan.e_parent[e] == root;
      }
      kid_rptr[vi + 1] = nr;
    }
    for (int64_t e = 0; e < NE; ++e) kid_eptr[e + 1] += kid_eptr[e];
    for (int64_t vi = 0; vi < NV; ++vi) kid_rptr[vi + 1] += kid_rptr[vi];
    kid_elist.resize(kid_eptr[NE]);
    kid_rlist.resize(kid_rptr[NV]);
    auto by_child = [&](int64_t a, int64_t b) { return plan.e_child[a] < plan.e_child[b]; };
#pragma omp parallel for schedule(static)
    for (int64_t vi = 0; vi < NV; ++vi) {
      const int root = part[plan.order[vi]];
      int64_t *rl = kid_rlist.data() + kid_rptr[vi];
      int nr = 0;
      for (int64_t e = plan.e_ptr[vi]; e < plan.e_ptr[vi + 1]; ++e) {
        int64_t *el = kid_elist.data() + kid_eptr[e];
        int nk = 0;
        for (int64_t f = plan.e_ptr[vi]; f < plan.e_ptr[vi + 1]; ++f)
          if (plan.e_parent[f] == plan.e_child[e]) el[nk++] = f;
        std::sort(el, el + nk, by_child);
        if (plan.e_parent[e] == root) rl[nr++] = e;
      }
      std::sort(rl, rl + nr, by_child);
    }
  }
  // children (edge indices, ascending child id) of node x of tree vi: the root, or the child
  // node of the tree's edge into x
  auto children_of = [&](int64_t vi, int x, int64_t *outv) -> int {
    const int64_t *b, *e;
    if (x == part[plan.order[vi]]) {
      b = kid_rlist.data() + kid_rptr[vi];
      e = kid_rlist.data() + kid_rptr[vi + 1];
    } else {
      const int64_t in = edge_into(vi, x);
      if (in < 0) return 0;
      b = kid_elist.data() + kid_eptr[in];
      e = kid_elist.data() + kid_eptr[in + 1];
    }
    int n = 0;
    for (const int64_t *q = b; q < e; ++q) outv[n++] = *q;
    return n;
  };
  lap("children index");

  // source buffer kind of every edge: the owner sends from its embeddings, a requester forwards
  // from its halo, a pure relay from its relay staging
  std::vector<int8_t> src_kind(NE);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < NE; ++e) {
    const int64_t u = plan.order[e_vidx[e]];
    const int p = plan.e_parent[e];
    src_kind[e] = p == part[u] ? K_EMB : (halo_pos(rel, u, p) >= 0 ? K_HALO : K_RELAY);
  }

  // NVSwitch multicast (the switch-level form of communication fusion,
  // P:1057-1065): single-stage plans only, every vertex requested by >= mc_min_fanout GPUs is
  // sent once, by its owner, with multimem stores into the multicast region every GPU binds at
  // the same offset (row mc_off[s] + j: the j-th such vertex of owner s in ascending id), then
  // each requester copies it from its own region into its halo row (unpack, local HBM)
  std::vector<uint8_t> mc_v(NV, 0);
  L.mc_rows.assign(m, 0);
  L.mc_off.assign(m + 1, 0);
  if (mc_min_fanout > 0 && K == 1) {
    for (int64_t vi = 0; vi < NV; ++vi) {
      const int64_t u = plan.order[vi];
      if (rel.d_ptr[u + 1] - rel.d_ptr[u] >= mc_min_fanout) {
        mc_v[vi] = 1;
        ++L.mc_rows[part[u]];
      }
    }
    for (int d = 0; d < m; ++d) L.mc_off[d + 1] = L.mc_off[d] + L.mc_rows[d];
  }
  L.mc_total = L.mc_off[m];

  // Leaf split (relay plans): a forward delivery that no later stage forwards (the edge's child
  // has no children in the tree) is needed only by its receiver, so it need not finish before
  // the next stage starts.  Such deliveries count on a counter block of their own that no stage
  // waits on, and their items come after the forwarded deliveries of the same stage: stage k+1's
  // items wait only for stage k's forwarded rows, and the leaves of stage k fill the time the
  // slowest CTA's forwarded rows take to land (the stage boundary).  Stage 1 (option 2) by edge,
  // or by row with fan-out items: one fan-out item stores a row into all its first hops, so the
  // row is "forwarded" if any of its first hops forwards it.
  const bool split = leaf_split > 0 && K >= 2 && NB == 1;
  std::vector<uint8_t> leaf_e;
  if (split) {
    L.leaf_block = 1;
    leaf_e.assign(NE, 0);
    std::vector<uint8_t> row_feeds(NV, 0);
    for (int64_t vi = 0; vi < NV; ++vi)
      for (int64_t e = plan.e_ptr[vi]; e < plan.e_ptr[vi + 1]; ++e)
        if (plan.e_stage[e] == 1 && kid_eptr[e + 1] > kid_eptr[e]) row_feeds[vi] = 1;
    // (stage 1 by row only with fan-out items; per-pair COPY groups split by edge)
    for (int64_t e = 0; e < NE; ++e)
      leaf_e[e] = plan.e_stage[e] == 1 && leaf_split < 2 ? 0
                  : plan.e_stage[e] == 1 && with_fanout   ? !row_feeds[e_vidx[e]]
                                                          : kid_eptr[e + 1] == kid_eptr[e];
  }
  auto fwd_block = [&](int64_t e) -> int {
    return split ? (leaf_e[e] ? L.leaf_block : 0) : blk_of[e_vidx[e]];
  };
  lap("blocks/child_pos/kinds");
  // ---- forward relay staging rows: contiguous per (receiver c, stage k, sender p, src kind) ----
  std::vector<int64_t> relay_row(NE, -1);
  {
    std::vector<Entry> rel_e;
    for (int64_t e = 0; e < NE; ++e)
      if (child_pos[e] < 0)
        rel_e.push_back({pack_key(plan.e_child[e], plan.e_stage[e], plan.e_parent[e],
                                  src_kind[e], 0),
                         e_vidx[e], e, e_vidx[e]});
    __gnu_parallel::sort(rel_e.begin(), rel_e.end(), [](const Entry &a, const Entry &b) {
      return a.key != b.key ? a.key < b.key : a.sort2 < b.sort2;
    });
    for (const Entry &x : rel_e) relay_row[x.edge] = L.n_relay[plan.e_child[x.edge]]++;
    L.n_relay_edges = (int64_t)rel_e.size();
  }

  auto flush_group = [&](std::vector<DevGroup> &groups, DevGroup g, const std::vector<int64_t> &src,
                         const std::vector<int64_t> &dst) {
    g.n_rows = (int64_t)dst.size();
    bool src_contig = !src.empty(), dst_contig = true;
    for (size_t i = 1; i < dst.size(); ++i) {
      if (dst[i] != dst[0] + (int64_t)i) dst_contig = false;
    }
    for (size_t i = 1; i < src.size(); ++i) {
      if (src[i] != src[0] + (int64_t)i) src_contig = false;
    }
    if (!src.empty()) {
      g.src_base = src[0];
      if (src_contig) {
        g.src_idx = -1;
      } else {
        g.src_idx = (int64_t)L.idx.size();
        for (int64_t v : src) L.idx.push_back((int32_t)v);
      }
    } else {
      g.src_idx = -1;
      g.src_base = 0;
    }
    g.dst_base = dst[0];
    if (dst_contig) {
      g.dst_idx = -1;
    } else {
      g.dst_idx = (int64_t)L.idx.size();
      for (int64_t v : dst) L.idx.push_back((int32_t)v);
    }
    groups.push_back(g);
  };

  auto base_group = [&](int op, int dir, int exec, int dst, int stage) {
    DevGroup g;
    std::memset(&g, 0, sizeof(g));
    g.op = op;
    g.dir = dir;
    g.exec_rank = exec;
    g.dst_rank = dst;
    g.stage = stage;
    g.sig_ctr = -1;
    g.ready_rank = -1;
    g.src_idx = g.dst_idx = -1;
    g.term_ptr = -1;
    return g;
  };

  lap("relay rows");
  // ---- forward groups: key (k, p, c, src_kind, dst_kind), rows sorted by destination row ----
  {
    std::vector<Entry> ent(NE);
    std::vector<int64_t> srow(NE), drow(NE);
    std::vector<uint8_t> keep(NE, 1);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < NE; ++e) {
      if (mc_v[e_vidx[e]]) {  // multicast vertex: its rows leave by the multicast groups
        keep[e] = 0;
        continue;
      }
      const int64_t vi = e_vidx[e];
      const int64_t u = plan.order[vi];
      const int p = plan.e_parent[e], c = plan.e_child[e], k = plan.e_stage[e];
      const int sk = src_kind[e];
      if (sk == K_EMB)
        srow[e] = loc[u];
      else if (sk == K_HALO)
        srow[e] = halo_pos(rel, u, p);
      else
        srow[e] = relay_row[edge_into(vi, p)];
      int dk;
      if (child_pos[e] >= 0) {
        dk = K_HALO;
        drow[e] = child_pos[e];
      } else {
        dk = K_RELAY;
        drow[e] = relay_row[e];
      }
      ent[e] = {pack_key_b(k, fwd_block(e), p, c, sk, dk), drow[e], e, vi};
    }
    if (L.mc_total > 0) {
      size_t w = 0;
      for (int64_t e = 0; e < NE; ++e)
        if (keep[e]) ent[w++] = ent[e];
      ent.resize(w);
    }
    __gnu_parallel::sort(ent.begin(), ent.end(), [](const Entry &a, const Entry &b) {
      return a.key != b.key ? a.key < b.key : a.sort2 < b.sort2;
    });
    std::vector<int64_t> src, dst;
    for (size_t i = 0; i < ent.size();) {
      size_t j = i;
      src.clear();
      dst.clear();
      while (j < ent.size() && ent[j].key == ent[i].key) {
        src.push_back(srow[ent[j].edge]);
        dst.push_back(drow[ent[j].edge]);
        ++j;
      }
      const uint64_t key = ent[i].key;
      const int k = key_stage(key), bl = key_block(key);
      const int p = (int)(key >> 16 & 0xFF), c = (int)(key >> 8 & 0xFF);
      DevGroup g = base_group(OP_COPY, DIR_FWD, p, c, k);
      g.block = bl;
      g.src_kind = (int)(key >> 4 & 0xF);
      g.dst_kind = (int)(key & 0xF);
      flush_group(L.groups, g, src, dst);
      L.rows_at(DIR_FWD, k, p, c, bl) += (int64_t)dst.size();
      i = j;
    }
    // multicast: per owner s one send group (its multicast vertices' embedding rows, ascending
    // id, into region rows mc_off[s] ..), then per (receiver d, owner s) one unpack group (region
    // rows of the s-vertices d requested -> d's halo rows), stage 2: after every send
    if (L.mc_total > 0) {
      std::vector<std::vector<int64_t>> mcv(m);  // multicast vertices of each owner, ascending
      for (int64_t vi = 0; vi < NV; ++vi)
        if (mc_v[vi]) mcv[part[plan.order[vi]]].push_back(plan.order[vi]);
      for (auto &v : mcv) std::sort(v.begin(), v.end());
      L.mc_begin = (int)L.groups.size();
      for (int s = 0; s < m; ++s) {
        if (mcv[s].empty()) continue;
        src.clear();
        dst.clear();
        for (size_t j = 0; j < mcv[s].size(); ++j) {
          src.push_back(loc[mcv[s][j]]);
          dst.push_back(L.mc_off[s] + (int64_t)j);
        }
        DevGroup g = base_group(OP_COPY, DIR_FWD, s, s, 1);
        g.src_kind = K_EMB;
        g.dst_kind = K_MCAST;
        flush_group(L.groups, g, src, dst);
      }
      for (int d = 0; d < m; ++d)
        for (int s = 0; s < m; ++s) {
          if (s == d || mcv[s].empty()) continue;
          src.clear();
          dst.clear();
          for (size_t j = 0; j < mcv[s].size(); ++j) {
            const int32_t pos = halo_pos(rel, mcv[s][j], d);
            if (pos < 0) continue;  // (fan-out below m - 1: d did not ask for this one)
            src.push_back(L.mc_off[s] + (int64_t)j);
            dst.push_back(pos);
          }
          if (dst.empty()) continue;
          DevGroup g = base_group(OP_COPY, DIR_FWD, d, d, 2);
          g.src_kind = K_MCUC;
          g.dst_kind = K_HALO;
          g.block = s;  // (the owner whose multicast rows it unpacks; see the waits below)
          flush_group(L.groups, g, src, dst);
        }
      L.mc_end = (int)L.groups.size();
    }
    L.n_fwd_groups = (int)L.groups.size();
  }

  lap("forward groups");
  // ---- backward pushes: key (b, c, p, sig) ----
  {
    // term signature of c's value for the vertex of edge e (c = child of e)
    std::vector<int8_t> sig(NE);
    std::vector<int8_t> nchild(NE, 0);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < NE; ++e) {
      const int64_t vi = e_vidx[e];
      int nc = 0;
      for (int64_t f = plan.e_ptr[vi]; f < plan.e_ptr[vi + 1]; ++f)
        if (plan.e_parent[f] == plan.e_child[e]) ++nc;
      nchild[e] = (int8_t)nc;
      const bool own = child_pos[e] >= 0;
      sig[e] = (own && nc == 0) ? 0 : (!own && nc == 1) ? 1 : 2;
    }
    std::vector<Entry> ent(NE);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < NE; ++e) {
      const int b = K - plan.e_stage[e] + 1;
      const int64_t sort2 = sig[e] == 0 ? (int64_t)child_pos[e] : plan.order[e_vidx[e]];
      ent[e] = {pack_key_b(b, blk_of[e_vidx[e]], plan.e_child[e], plan.e_parent[e], sig[e], 0),
                sort2, e, e_vidx[e]};
    }
    __gnu_parallel::sort(ent.begin(), ent.end(), [](const Entry &a, const Entry &b) {
      return a.key != b.key ? a.key < b.key : a.sort2 < b.sort2;
    });
    lap("  bwd sig + sort");
    // children of node x in tree vi, ascending id -> their edge indices
    auto children_edges = children_of;
    // RED rows of every owner: (loc, vertex index) ascending
    std::vector<std::vector<std::pair<int64_t, int64_t>>> red_rows(m);
    for (int64_t vi = 0; vi < NV; ++vi) {
      const int64_t u = plan.order[vi];
      if (plan.e_ptr[vi + 1] > plan.e_ptr[vi]) red_rows[part[u]].push_back({loc[u], vi});
    }
    for (auto &rr : red_rows) std::sort(rr.begin(), rr.end());

    // Slot rows on the parent in the order the parent READS them: every slot row is an operand
    // of exactly one fold (or forwarding copy) of its parent x — x's own push of that vertex
    // (push groups in execution order, rows in group order) or x's RED (loc order) — which takes
    // its children's slots in ascending child id.  So a fold reads its slot operands as runs of
    // consecutive rows (few bulk copies per item) and a relay with one child forwards a
    // contiguous slot range; the children's pushes scatter their rows into it (destination index
    // lists).  Measured against slots contiguous per push group (A/B on one B200, bwd ms):
    // Web-Google ring 2.08 -> 1.92, Reddit dgx1_like 1.24 -> 1.18, Web-Google dgx1_like
    // 1.82 -> 1.91; against slots grouped per (consumer group, child) with pushes in consumer
    // order: 2.09 / 1.20 / 1.90.
    lap("  bwd red_rows");
    std::vector<int64_t> slot_row(NE, -1);
    {
      int64_t chs[kMaxRanks];
      for (const Entry &x : ent) {  // (the children of edge x's child node: its kid list)
        const int64_t kb = kid_eptr[x.edge], ke = kid_eptr[x.edge + 1];
        if (kb == ke) continue;
        int64_t &ns = L.n_slot[plan.e_child[x.edge]];
        for (int64_t q = kb; q < ke; ++q) slot_row[kid_elist[q]] = ns++;
      }
      for (int s = 0; s < m; ++s)
        for (auto &r : red_rows[s]) {
          const int n = children_edges(r.second, s, chs);
          for (int t = 0; t < n; ++t) slot_row[chs[t]] = L.n_slot[s]++;
        }
    }

    lap("  bwd slot rows");
    std::vector<int64_t> src, dst;
    int64_t ch[kMaxRanks];
    for (size_t i = 0; i < ent.size();) {
      size_t j = i;
      while (j < ent.size() && ent[j].key == ent[i].key) ++j;
      const uint64_t key = ent[i].key;
      const int b = key_stage(key), bl = key_block(key);
      const int c = (int)(key >> 16 & 0xFF), p = (int)(key >> 8 & 0xFF);
      const int s = (int)(key >> 4 & 0xF);
      src.clear();
      dst.clear();
      DevGroup g = base_group(s == 2 ? OP_FOLD : OP_COPY, DIR_BWD, c, p, b);
      g.block = bl;
      g.dst_kind = K_SLOT;
      if (s == 2) {
        g.term_ptr = (int64_t)L.term_ptr.size();
        L.term_ptr.push_back((int64_t)L.terms.size());
      }
      for (size_t q = i; q < j; ++q) {
        const int64_t e = ent[q].edge;
        dst.push_back(slot_row[e]);
        if (s == 0) {
          src.push_back(child_pos[e]);
        } else if (s == 1) {
          src.push_back(slot_row[kid_elist[kid_eptr[e]]]);
        } else {
          if (child_pos[e] >= 0) L.terms.push_back((uint32_t)child_pos[e]);
          for (int64_t q = kid_eptr[e]; q < kid_eptr[e + 1]; ++q)
            L.terms.push_back(kTermSlot | (uint32_t)slot_row[kid_elist[q]]);
          L.term_ptr.push_back((int64_t)L.terms.size());
        }
      }
      g.src_kind = s == 0 ? K_HGRAD : K_SLOT;
      flush_group(L.groups, g, src, dst);
      L.rows_at(DIR_BWD, b, c, p, bl) += (int64_t)(j - i);
      i = j;
    }

    lap("  bwd push groups");
    // ---- RED: owner folds its slots into emb_grad, ascending child id, stage K + 1 ----
    for (int bl = 0; bl < NB; ++bl)
    for (int s = 0; s < m; ++s) {
      std::vector<std::pair<int64_t, int64_t>> rows;  // (loc, vidx) of block bl
      for (const auto &r : red_rows[s])
        if (blk_of[r.second] == bl) rows.push_back(r);
      if (rows.empty()) continue;
      DevGroup g = base_group(OP_FOLD, DIR_BWD, s, s, K + 1);
      g.block = bl;
      g.dst_kind = K_EGRAD;
      g.fold_init = 1;
      g.term_ptr = (int64_t)L.term_ptr.size();
      L.term_ptr.push_back((int64_t)L.terms.size());
      dst.clear();
      src.clear();
      for (auto &r : rows) {
        dst.push_back(r.first);
        const int n = children_edges(r.second, s, ch);
        for (int t = 0; t < n; ++t) L.terms.push_back(kTermSlot | (uint32_t)slot_row[ch[t]]);
        L.term_ptr.push_back((int64_t)L.terms.size());
      }
      flush_group(L.groups, g, src, dst);
    }
  }

  lap("backward pushes + RED");
  // ---- signals and waits (the ready/done protocol of §6.1) ----
  // wait lists per (dir, stage, exec, block): every in-peer's counter of the previous stage of
  // the same vertex block
  std::map<std::tuple<int, int, int, int>, std::pair<int32_t, int32_t>> wait_lists;
  auto get_waits = [&](int dir, int stage_prev, int r, int bl) {
    auto key = std::make_tuple(dir, stage_prev, r, bl);
    auto it = wait_lists.find(key);
    if (it != wait_lists.end()) return it->second;
    const int32_t off = (int32_t)L.waits.size();
    for (int s = 0; s < m; ++s) {
      const int64_t rows = L.rows(dir, stage_prev, s, r, bl);
      if (rows > 0) L.waits.push_back({(int32_t)ctr_index(dir, stage_prev, s, bl), 0, rows});
    }
    auto v = std::make_pair(off, (int32_t)L.waits.size() - off);
    wait_lists[key] = v;
    return v;
  };
  for (DevGroup &g : L.groups) {
    if (g.dst_rank != g.exec_rank) {
      g.sig_ctr = (int32_t)ctr_index(g.dir, g.stage, g.exec_rank, g.block);
      g.ready_rank = g.dst_rank;
    }
    bool reads_inflight;
    if (g.dir == DIR_FWD)
      reads_inflight = g.src_kind != K_EMB;
    else
      reads_inflight = g.op == OP_FOLD || g.src_kind == K_SLOT;
    if (reads_inflight && g.stage >= 2) {
      // (leaf split: every forwarded row arrived on the previous stage's non-leaf counters)
      auto w = get_waits(g.dir, g.stage - 1, g.exec_rank,
                         split && g.dir == DIR_FWD ? 0 : g.block);
      g.wait_off = w.first;
      g.wait_n = w.second;
    }
  }
  // multicast groups: a send signals the multicast done counter of its owner (one multimem
  // reduction reaches every GPU's copy) and writes into every peer's region (all ready words);
  // an unpack waits on the owner's multicast counter in this GPU's own region
  // an unpack signals its own GPU's stage-2 counter of the owner s (arrival waits, R25: the rows
  // of s that came by multicast are in the halo once it reaches its target); its wait entry is
  // kept for dgcl_stream_wait_arrival
  L.mc_unpack_wait.assign((size_t)m * m, -1);
  for (int gi = L.mc_begin; gi < L.mc_end; ++gi) {
    DevGroup &g = L.groups[gi];
    g.wait_off = 0;
    g.wait_n = 0;
    if (g.dst_kind == K_MCAST) {
      g.sig_ctr = (int32_t)(kMcCtrBase + g.exec_rank);
      g.ready_rank = kReadyAll;
    } else {
      const int s_owner = g.block;
      g.block = 0;
      g.wait_off = (int32_t)L.waits.size();
      g.wait_n = 1;
      L.waits.push_back({(int32_t)(kMcCtrBase + s_owner), 0, L.mc_rows[s_owner]});
      g.sig_ctr = (int32_t)ctr_index(DIR_FWD, 2, s_owner, 0);
      L.mc_unpack_wait[(size_t)g.exec_rank * m + s_owner] = (int32_t)L.waits.size();
      L.waits.push_back({g.sig_ctr, 0, g.n_rows});
    }
  }
  // per-rank READY and forward-completion WAIT groups (used by per-rank programs only)
  for (int r = 0; r < m; ++r) {
    DevGroup g = base_group(OP_READY, DIR_FWD, r, r, 0);
    L.groups.push_back(g);
  }
  for (int r = 0; r < m; ++r) {
    DevGroup g = base_group(OP_WAIT, DIR_FWD, r, r, K + 1);
    g.wait_off = (int32_t)L.waits.size();
    for (int k = 1; k <= K; ++k)
      for (int bl = 0; bl < (split ? L.leaf_block + 1 : NB); ++bl)
        for (int s = 0; s < m; ++s) {
          const int64_t rows = L.rows(DIR_FWD, k, s, r, bl);
          if (rows > 0) L.waits.push_back({(int32_t)ctr_index(DIR_FWD, k, s, bl), 0, rows});
        }
    g.wait_n = (int32_t)L.waits.size() - g.wait_off;
    L.groups.push_back(g);
  }
  lap("signals/waits");
  // ---- loopback direct reduce (single-stage plans only) ----
  // When every virtual rank lives on one device the owner can read its requesters' halo-gradient
  // rows in place: emb_grad[loc u] = ((emb_grad[loc u] + G_c1[pos]) + G_c2[pos]) + ..., c
  // ascending — the same fold, terms and order as push + RED, without the slot round trip.
  L.direct_begin = (int)L.groups.size();
  if (K <= 1) {
    for (int s = 0; s < m; ++s) {
      std::vector<std::pair<int64_t, int64_t>> rows;  // (loc, u)
      for (int64_t vi = 0; vi < NV; ++vi) {
        const int64_t u = plan.order[vi];
        if (part[u] == s) rows.push_back({loc[u], u});
      }
      if (rows.empty()) continue;
      std::sort(rows.begin(), rows.end());
      DevGroup g = base_group(OP_FOLD, DIR_BWD, s, s, 1);
      g.dst_kind = K_EGRAD;
      g.fold_init = 1;
      g.term_mode = kTermRankHgrad;
      g.term_ptr = (int64_t)L.term_ptr.size();
      L.term_ptr.push_back((int64_t)L.terms.size());
      std::vector<int64_t> dst, src;
      for (auto &r : rows) {
        dst.push_back(r.first);
        for (int64_t q = rel.d_ptr[r.second]; q < rel.d_ptr[r.second + 1]; ++q)
          L.terms.push_back(((uint32_t)rel.d_gpu[q] << 28) | ((uint32_t)rel.d_pos[q] & kTermRowMask));
        L.term_ptr.push_back((int64_t)L.terms.size());
      }
      flush_group(L.groups, g, src, dst);
    }
  }
  L.direct_end = (int)L.groups.size();
  lap("direct reduce");
  // ---- loopback atomic backward (ablation, single-stage plans only) ----
  // The paper's "Atomic" baseline (§6.2, Table 9): every requester adds
  // its halo-gradient rows straight into the owner's rows with atomic reductions, one group per
  // (requester c, owner p), rows in c's halo order (consecutive source rows).  Same sum, but the
  // order of the adds is whatever the hardware makes it: not reproducible bit for bit.
  if (K <= 1 && with_atomic) {
    std::vector<std::vector<std::pair<int64_t, int64_t>>> pairs((size_t)m * m);  // (pos_c, loc)
    for (int64_t vi = 0; vi < NV; ++vi) {
      const int64_t u = plan.order[vi];
      for (int64_t q = rel.d_ptr[u]; q < rel.d_ptr[u + 1]; ++q)
        pairs[(size_t)rel.d_gpu[q] * m + part[u]].push_back({rel.d_pos[q], loc[u]});
    }
    for (int c = 0; c < m; ++c)
      for (int p = 0; p < m; ++p) {
        auto &v = pairs[(size_t)c * m + p];
        if (v.empty()) continue;
        std::sort(v.begin(), v.end());
        DevGroup g = base_group(OP_COPY, DIR_BWD, c, p, 1);
        g.src_kind = K_HGRAD;
        g.dst_kind = K_EGRAD;
        g.atomic_add = 1;
        std::vector<int64_t> src, dst;
        for (auto &x : v) {
          src.push_back(x.first);
          dst.push_back(x.second);
        }
        flush_group(L.groups, g, src, dst);
      }
  }
  L.atomic_end = (int)L.groups.size();
  // ---- forward stage 1 as fan-out groups (one per owner) ----
  // Every stage-1 tree edge leaves the owner (the root), so stage 1 is "each owner sends each of
  // its rows to the requesters of that row" (P:1458-1462 packs one (d_i, d_j) tuple at a time).
  // A fan-out group reads each embedding row ONCE and stores it into all its first-hop receivers
  // (halo row, or relay staging for a forwarding GPU) — the kernel-level form of the paper's
  // communication fusion: HBM reads drop from one per delivery to one per row.
  // Rows are the owner's local rows in loc order (consecutive sources: one bulk copy per item);
  // dests per row in ascending receiver id, as word pairs in the terms pool: (receiver << 28 |
  // relay bit | destination row, source row) — the executor maps (pair, chunk) to threads.
  if (with_fanout) {
    int64_t N = (int64_t)loc.size();
    std::vector<int64_t> vi_of(N, -1);
    for (int64_t vi = 0; vi < NV; ++vi) vi_of[plan.order[vi]] = vi;
    std::vector<std::vector<int64_t>> rows_of(m);  // owner -> vertices in loc order
    for (int64_t u = 0; u < N; ++u) rows_of[part[u]].push_back(u);
    bool fits = true;
    std::vector<std::pair<int, uint32_t>> ds;
    // (leaf split of stage 1: the owners' forwarded rows first, then their leaf rows; a group
    // keeps all the owner's rows, the other class's rows without receivers)
    const int n_cls = split && leaf_split >= 2 ? 2 : 1;
    for (int cls = 0; cls < n_cls && fits; ++cls)
    for (int p = 0; p < m && fits; ++p) {
      DevGroup g = base_group(OP_FANOUT, DIR_FWD, p, p, 1);
      const int fblock = n_cls == 2 && cls == 1 ? L.leaf_block : 0;
      g.block = fblock;
      g.src_kind = K_EMB;
      g.dst_kind = K_HALO;
      g.n_rows = (int64_t)rows_of[p].size();
      g.src_base = 0;
      g.dst_base = 0;
      g.sig_ctr = (int32_t)ctr_index(DIR_FWD, 1, p, fblock);
      g.ready_rank = kReadyAll;
      g.term_ptr = (int64_t)L.term_ptr.size();
      const size_t t_begin = L.terms.size();
      L.term_ptr.push_back((int64_t)L.terms.size());
      for (int64_t u : rows_of[p]) {
        const int64_t vi = vi_of[u];
        if (vi >= 0) {
          ds.clear();
          for (int64_t e = plan.e_ptr[vi]; e < plan.e_ptr[vi + 1]; ++e) {
            if (plan.e_parent[e] != p) continue;
            if (n_cls == 2 && fwd_block(e) != fblock) continue;
            const int c = plan.e_child[e];
            const int64_t row = child_pos[e] >= 0 ? child_pos[e] : relay_row[e];
            if (row > (int64_t)kFanRowMask) fits = false;
            ds.push_back({c, ((uint32_t)c << 28) | (child_pos[e] >= 0 ? 0u : kFanRelay) |
                                 ((uint32_t)row & kFanRowMask)});
          }
          std::sort(ds.begin(), ds.end());
          for (auto &d : ds) {
            L.terms.push_back(d.second);
            L.terms.push_back((uint32_t)loc[u]);
          }
        }
        L.term_ptr.push_back((int64_t)L.terms.size());
      }
      if (L.terms.size() > t_begin) L.groups.push_back(g);
    }
    if (!fits) L.groups.resize(L.atomic_end);  // rows beyond the 27-bit dest field: per-pair groups
  }
  L.fanout_end = (int)L.groups.size();
  lap("atomic/fanout groups");
  // ---- loopback tree-order backward (relay plans) ----
  // With every virtual rank on one device the owner can evaluate the reversed plan's whole fold
  // for its row in one pass: the staged backward computes val_c(u) = ((own_c + val(y1)) +
  // val(y2)) ... bottom-up along T_u and the owner emb_grad = ((L + val(c1)) +
  // val(c2)) ...; here the same expression, same operands, same association, is one postfix
  // program per owner row over the requesters' halo-gradient rows (kTermRankTree), so the
  // result is bit-identical to the staged pushes without their slot round trips and stage
  // barriers.  (The multi-GPU form, and loopback with direct_reduce = 0, run the stages.)
  if (K >= 2) {
    auto kids = children_of;
    bool fits = true;
    int depth = 0, max_depth = 0;
    // postfix of val(x) for vertex vi: own(x) (if x requested u), then each child ascending,
    // an add after every value but the first; an add is counted on the operand word just
    // emitted (every add follows an operand or another add)
    auto add_after_last = [&]() {
      const uint32_t w = L.terms.back();
      const uint32_t a = ((w >> kTreeAddShift) & 15u) + 1;
      if (a > 15) fits = false;
      L.terms.back() = (w & ~(15u << kTreeAddShift)) | ((a & 15u) << kTreeAddShift);
      --depth;
    };
    std::function<void(int64_t, int)> emit = [&](int64_t vi, int x) {
      const int64_t u = plan.order[vi];
      int64_t ch[kMaxRanks];
      const int n = kids(vi, x, ch);
      const int32_t pos = halo_pos(rel, u, x);
      bool have = false;
      if (pos >= 0) {
        if ((uint32_t)pos > kTreeRowMask) fits = false;
        L.terms.push_back(((uint32_t)x << 28) | ((uint32_t)pos & kTreeRowMask));
        max_depth = std::max(max_depth, ++depth);
        have = true;
      }
      for (int t = 0; t < n; ++t) {
        emit(vi, plan.e_child[ch[t]]);
        if (have) add_after_last();
        have = true;
      }
    };
    std::vector<std::vector<std::pair<int64_t, int64_t>>> rows_of(m);  // (loc, vi)
    for (int64_t vi = 0; vi < NV; ++vi)
      if (plan.e_ptr[vi + 1] > plan.e_ptr[vi]) rows_of[part[plan.order[vi]]].push_back({loc[plan.order[vi]], vi});
    const size_t t_begin = L.terms.size(), p_begin = L.term_ptr.size();
    for (int s = 0; s < m && fits; ++s) {
      auto &rows = rows_of[s];
      if (rows.empty()) continue;
      std::sort(rows.begin(), rows.end());
      DevGroup g = base_group(OP_FOLD, DIR_BWD, s, s, 1);
      g.dst_kind = K_EGRAD;
      g.fold_init = 1;
      g.term_mode = kTermRankTree;
      g.term_ptr = (int64_t)L.term_ptr.size();
      L.term_ptr.push_back((int64_t)L.terms.size());
      std::vector<int64_t> src, dst;
      int64_t ch[kMaxRanks];
      for (auto &r : rows) {
        dst.push_back(r.first);
        const int n = kids(r.second, s, ch);
        for (int t = 0; t < n; ++t) {  // ((L + val(c1)) + val(c2)) ...: L is the stack bottom
          depth = 1;
          emit(r.second, plan.e_child[ch[t]]);
          add_after_last();
        }
        L.term_ptr.push_back((int64_t)L.terms.size());
      }
      flush_group(L.groups, g, src, dst);
    }
    if (!fits || max_depth > kTreeMaxDepth) {  // too deep for the register stack: staged form
      L.groups.resize(L.fanout_end);
      L.terms.resize(t_begin);
      L.term_ptr.resize(p_begin);
    }
  }
  L.tree_end = (int)L.groups.size();
  lap("tree programs");
  L.seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
}

namespace {

// Staged FOLD item (bulk-copy executor): operand rows [0, rows) of the stage are the
// destination rows the fold starts from (fold_init), then every term's source row, sorted by
// (buffer kind, rank, row) so that consecutive rows form one segment = one bulk copy.  With the
// harness's halo order (owner, id) an owner's requesters' rows are consecutive, so a loopback
// reduce item needs one segment per requesting rank.  The terms keep their order; sterms only
// says where each one's row sits in the stage.
constexpr int64_t kMinSegmentRows = 4;  // staged FOLD groups: average operand rows per segment

void stage_fold_item(const Lowered &low, const DevGroup &g, DevItem *it, std::vector<DevRun> *runs,
                     std::vector<uint32_t> *sterms) {
  struct Ref {
    int32_t key;  // (kind << 8) | rank
    int32_t row;
    int64_t t;    // term index (or -1 - r for the destination row r)
  };
  std::vector<Ref> refs;
  auto drow = [&](int64_t r) {
    return g.dst_idx >= 0 ? (int64_t)low.idx[g.dst_idx + r] : g.dst_base + r;
  };
  const int64_t rb = it->tp - g.term_ptr;
  const int64_t seg0 = (int64_t)runs->size();
  if (g.fold_init) {
    for (int64_t r = 0; r < it->rows;) {  // destination rows: operand rows 0 .. rows-1
      int64_t e = r + 1;
      while (e < it->rows && drow(rb + e) == drow(rb + e - 1) + 1) ++e;
      runs->push_back({(int32_t)drow(rb + r), (g.dst_kind << 8) | g.dst_rank, (int32_t)(e - r),
                       (int32_t)r});
      r = e;
    }
  }
  for (int64_t t = it->t0; t < it->t0 + it->nterms; ++t) {
    const uint32_t x = low.terms[t];
    Ref f;
    if (g.term_mode == kTermRankTree) {
      f.key = (K_HGRAD << 8) | (int32_t)(x >> 28);
      f.row = (int32_t)(x & kTreeRowMask);
    } else if (g.term_mode == kTermRankHgrad) {
      f.key = (K_HGRAD << 8) | (int32_t)(x >> 28);
      f.row = (int32_t)(x & kTermRowMask);
    } else if (x & kTermSlot) {
      f.key = (K_SLOT << 8) | g.exec_rank;
      f.row = (int32_t)(x & ~kTermSlot);
    } else {
      f.key = (K_HGRAD << 8) | g.exec_rank;
      f.row = (int32_t)x;
    }
    f.t = t;
    refs.push_back(f);
  }
  std::sort(refs.begin(), refs.end(), [](const Ref &a, const Ref &b) {
    return a.key != b.key ? a.key < b.key : a.row < b.row;
  });
  const int64_t base = g.fold_init ? it->rows : 0;
  const int64_t st0 = (int64_t)sterms->size();
  sterms->resize(st0 + it->nterms);
  for (size_t a = 0; a < refs.size();) {
    size_t e = a + 1;
    while (e < refs.size() && refs[e].key == refs[a].key && refs[e].row == refs[e - 1].row + 1) ++e;
    runs->push_back({refs[a].row, refs[a].key, (int32_t)(e - a), (int32_t)(base + (int64_t)a)});
    a = e;
  }
  for (size_t a = 0; a < refs.size(); ++a)  // (tree programs keep each term's adds)
    (*sterms)[st0 + (refs[a].t - it->t0)] =
        (uint32_t)(base + (int64_t)a) |
        (g.term_mode == kTermRankTree ? low.terms[refs[a].t] & (15u << kTreeAddShift) : 0u);
  it->flags |= kItemStaged;
  it->src = ((int64_t)((int64_t)runs->size() - seg0) << kSegShift) | seg0;
  it->t0 = st0;
}

}  // namespace

ItemLimits item_limits(const TmaGeometry &g, int64_t item_bytes, int64_t min_items) {
  ItemLimits l;
  l.min_items = min_items;
  l.operand_bytes = std::min<int64_t>(item_bytes, g.stage_bytes - kStageHdrBytes);
  l.max_rows = std::min<int64_t>(kMaxItemRows, g.max_item_rows);
  return l;
}

void build_items(const Lowered &low, const std::vector<int32_t> &gids, int64_t row_bytes,
                 const ItemLimits &lim, bool signal_all, const std::vector<uint8_t> &needed_ctr,
                 std::vector<DevItem> *items, std::vector<DevRun> *runs,
                 int64_t direct_copy_rows, std::vector<uint32_t> *sterms) {
  runs->clear();
  if (sterms) sterms->clear();
  // An item is a row range whose gathered operands fit `item_bytes` (and one shared-memory stage
  // of the bulk-copy executor): a COPY row costs one row, a FOLD row (1 + #terms) rows.
  items->clear();
  const int64_t row16 = (row_bytes + 15) / 16 * 16;
  const int64_t cap = std::max<int64_t>(row16, lim.operand_bytes);
  size_t i = 0;
  std::vector<std::vector<int32_t>> bounds;  // per group of the stage: chunk start rows + end
  std::vector<uint8_t> staged;               // per group of the stage: FOLD items are staged
  // per group of the stage: OP_FANOUT items as row ranges [first, second) (runs of rows without
  // receivers between them are skipped, so items are not contiguous in the group's rows)
  std::vector<std::vector<std::pair<int64_t, int64_t>>> franges;
  std::vector<uint8_t> aligned;  // per group of the stage: bounds set jointly (source-aligned)
  // staged FOLD item: operand rows (destination rows of the fold start + one per term) and the
  // staged-term window share one stage; segments (<= one per operand row) fill one meta slot
  const int64_t stage_rows_cap = std::min<int64_t>(lim.max_rows, lim.operand_bytes / row16);
  auto staged_fits = [&](int64_t srows, int64_t nt) {
    return srows <= stage_rows_cap &&
           srows * row16 + (nt * 4 + 15) / 16 * 16 + 16 <= lim.operand_bytes;
  };
  auto src_row = [&](const DevGroup &h, int64_t r) -> int64_t {
    return h.src_idx >= 0 ? (int64_t)low.idx[h.src_idx + r] : h.src_base + r;
  };
  auto ascending_src = [&](const DevGroup &h) {
    for (int64_t r = 1; r < h.n_rows; ++r)
      if (src_row(h, r) <= src_row(h, r - 1)) return false;
    return true;
  };
  while (i < gids.size()) {
    // one stage (READY / WAIT are their own runs)
    const DevGroup &g0 = low.groups[gids[i]];
    size_t j = i;
    while (j < gids.size() && low.groups[gids[j]].stage == g0.stage &&
           low.groups[gids[j]].block == g0.block &&
           low.groups[gids[j]].op != OP_READY && low.groups[gids[j]].op != OP_WAIT &&
           g0.op != OP_READY && g0.op != OP_WAIT)
      ++j;
    if (j == i) j = i + 1;
    bounds.assign(j - i, std::vector<int32_t>());
    staged.assign(j - i, 0);
    franges.assign(j - i, {});
    size_t max_chunks = 0;
    // small stages: cut COPY items finer so that every co-resident CTA gets work (latency-bound
    // launches, e.g. the tiny config or the last relay stage), down to 4 rows per item
    int64_t copy_rows = 0;
    for (size_t q = i; q < j; ++q)
      if (low.groups[gids[q]].op == OP_COPY) copy_rows += low.groups[gids[q]].n_rows;
    int64_t spread_rpi = lim.max_rows;
    if (lim.min_items > 0 && low.n_blocks == 1 && copy_rows < lim.min_items * lim.max_rows)
      spread_rpi = std::max<int64_t>(4, (copy_rows + lim.min_items - 1) / lim.min_items);
    auto copy_rpi = [&](int64_t spread) {
      // (lsu_gather: the source-row window shares the stage with the rows)
      const int64_t per_row = lim.lsu_gather ? row16 + 4 : row16;
      int64_t rpi = std::min<int64_t>(std::min(lim.max_rows, spread),
                                      std::max<int64_t>(1, (cap - (lim.lsu_gather ? 32 : 0)) / per_row));
      if (row16 <= kGather4MaxRowBytes && rpi >= 4) rpi = rpi / 4 * 4;
      return rpi;
    };
    // Forward COPY groups that read the same rank's embeddings (one per receiver) get item
    // boundaries at the SAME source rows: chunk c of every such group covers source rows
    // [B_c, B_c+1), and chunks are interleaved, so the copies of one row to its receivers run
    // close together and all but the first hit L2 (independent cuts drift apart over a long
    // launch: the Com-Orkut forward re-read 0.7 GB on top of its 1.6 GB of rows, ncu r1i).  A
    // cut falls where the first group of the set reaches `rpi` rows, so no item exceeds it.
    // Applied to rows <= 1 KB (the per-row gather regime): measured Web-Google-4 forward 0.345
    // -> 0.308 ms, Com-Orkut 1.62 -> 1.60, Web-Google-8 0.448 -> 0.445; the Reddit dim-602
    // forward, whose rows already come once from DRAM, lost 2 % to the smaller items.
    aligned.assign(j - i, 0);
    if (lim.align_sources && row16 <= kGather4MaxRowBytes) {
      // (groups whose sources come in short runs, < 4 rows on average — the per-row gather
      // regime; long runs already stream each row once)
      auto short_runs = [&](const DevGroup &h) {
        int64_t runs = 1;
        for (int64_t r = 1; r < h.n_rows; ++r) runs += src_row(h, r) != src_row(h, r - 1) + 1;
        return runs * 4 > h.n_rows;
      };
      auto alignable = [&](const DevGroup &h) {
        return h.op == OP_COPY && h.dir == DIR_FWD && h.src_kind == K_EMB && !h.atomic_add &&
               h.dst_kind != K_MCAST && h.n_rows > 0 && ascending_src(h) && short_runs(h);
      };
      const int64_t rpi = copy_rpi(spread_rpi);
      std::vector<uint8_t> can(j - i);  // alignable, evaluated once per group (O(rows))
      for (size_t q = i; q < j; ++q) can[q - i] = alignable(low.groups[gids[q]]) ? 1 : 0;
      for (size_t q = i; q < j; ++q) {
        const DevGroup &g = low.groups[gids[q]];
        if (aligned[q - i] || !can[q - i]) continue;
        // (groups of about the same size only: relay plans' first hops are very uneven, and a
        // dense group would cut a sparse one into many small items)
        std::vector<size_t> set;
        int64_t big = 0;
        for (size_t q2 = q; q2 < j; ++q2) {
          const DevGroup &h = low.groups[gids[q2]];
          if (!aligned[q2 - i] && h.exec_rank == g.exec_rank && can[q2 - i])
            big = std::max(big, h.n_rows);
        }
        for (size_t q2 = q; q2 < j; ++q2) {
          const DevGroup &h = low.groups[gids[q2]];
          if (!aligned[q2 - i] && h.exec_rank == g.exec_rank && can[q2 - i] &&
              4 * h.n_rows >= 3 * big)
            set.push_back(q2);
        }
        if (set.size() < 2) continue;
        std::vector<int64_t> ptr(set.size(), 0);
        for (size_t t = 0; t < set.size(); ++t) {
          aligned[set[t] - i] = 1;
          bounds[set[t] - i].assign(1, 0);
        }
        for (;;) {
          int64_t B = INT64_MAX;
          bool left = false;
          for (size_t t = 0; t < set.size(); ++t) {
            const DevGroup &h = low.groups[gids[set[t]]];
            if (ptr[t] >= h.n_rows) continue;
            left = true;
            if (ptr[t] + rpi < h.n_rows) B = std::min(B, src_row(h, ptr[t] + rpi));
          }
          if (!left) break;
          for (size_t t = 0; t < set.size(); ++t) {
            const DevGroup &h = low.groups[gids[set[t]]];
            int64_t lo = B == INT64_MAX ? h.n_rows : ptr[t], hi = h.n_rows;
            if (B != INT64_MAX)
              while (lo < hi) {  // first row whose source is >= B (sources ascending)
                const int64_t mid = (lo + hi) / 2;
                if (src_row(h, mid) < B) lo = mid + 1; else hi = mid;
              }
            ptr[t] = lo;
            bounds[set[t] - i].push_back((int32_t)lo);
          }
          if (B == INT64_MAX) break;
        }
      }
    }
    for (size_t q = i; q < j; ++q) {
      const DevGroup &g = low.groups[gids[q]];
      std::vector<int32_t> &b = bounds[q - i];
      if (aligned[q - i]) {
        max_chunks = std::max(max_chunks, b.size() - 1);
        continue;
      }
      b.push_back(0);
      if (g.op == OP_FOLD && sterms) {
        // staged: every row must fit a stage on its own
        bool ok = true;
        for (int64_t r = 0; r < g.n_rows && ok; ++r) {
          const int64_t nt = low.term_ptr[g.term_ptr + r + 1] - low.term_ptr[g.term_ptr + r];
          ok = staged_fits(nt + (g.fold_init ? 1 : 0), nt);
        }
        staged[q - i] = ok ? 1 : 0;
      }
      if (g.op == OP_COPY) {
        // rows per item; a multiple of 4 when gather4 may apply (its groups are padded to 4 rows)
        const int64_t rpi = copy_rpi(spread_rpi);
        for (int64_t r = rpi; r < g.n_rows; r += rpi) b.push_back((int32_t)r);
        b.push_back((int32_t)g.n_rows);
      } else if (g.op == OP_FOLD && staged[q - i]) {
        int64_t srows = 0, nt = 0;
        for (int64_t r = 0; r < g.n_rows; ++r) {
          const int64_t c = low.term_ptr[g.term_ptr + r + 1] - low.term_ptr[g.term_ptr + r];
          const int64_t add = c + (g.fold_init ? 1 : 0);
          if (r > b.back() && (!staged_fits(srows + add, nt + c) || r - b.back() >= kMaxFoldRows ||
                               nt + c > kMaxItemTerms)) {
            b.push_back((int32_t)r);
            srows = nt = 0;
          }
          srows += add;
          nt += c;
        }
        b.push_back((int32_t)g.n_rows);
        // staging pays when segments are long (one bulk copy each); operand rows scattered in
        // short runs (e.g. relay slots) are better gathered by the consumers' plain loads
        int64_t nseg = 0, nst = 0;
        std::vector<DevRun> trial_runs;
        std::vector<uint32_t> trial_st;
        for (size_t c = 0; c + 1 < b.size(); ++c) {
          DevItem t;
          std::memset(&t, 0, sizeof(t));
          t.rows = b[c + 1] - b[c];
          t.tp = g.term_ptr + b[c];
          t.t0 = low.term_ptr[t.tp];
          t.nterms = (int32_t)(low.term_ptr[t.tp + t.rows] - t.t0);
          t.dst = g.dst_idx >= 0 ? ~(g.dst_idx + b[c]) : g.dst_base + b[c];
          trial_runs.clear();
          trial_st.clear();
          stage_fold_item(low, g, &t, &trial_runs, &trial_st);
          nseg += (int64_t)trial_runs.size();
          nst += t.nterms + (g.fold_init ? t.rows : 0);
        }
        if (nst < kMinSegmentRows * nseg) {
          staged[q - i] = 0;
          b.assign(1, 0);
        }
      }
      if (g.op == OP_FOLD && !staged[q - i]) {
        int64_t acc = 0;
        for (int64_t r = 0; r < g.n_rows; ++r) {
          const int64_t slots = low.term_ptr[g.term_ptr + r + 1] - low.term_ptr[g.term_ptr + r] +
                                (g.fold_init ? 1 : 0);
          // FOLD operands are gathered by the consumers straight from memory (not staged): the
          // item is bounded by 4x the gathered bytes of a COPY item and by its tables
          const int64_t cost = slots * row16;
          const int64_t nt = low.term_ptr[g.term_ptr + r + 1] - low.term_ptr[g.term_ptr + b.back()];
          if (acc > 0 &&
              (acc + cost > 4 * cap || r - b.back() >= kMaxFoldRows || nt > kMaxItemTerms)) {
            b.push_back((int32_t)r);
            acc = 0;
          }
          acc += cost;
        }
        b.push_back((int32_t)g.n_rows);
      } else if (g.op == OP_FANOUT) {
        // the source rows of an item are consecutive (one bulk copy) and its operands — rows and
        // destination words — fit one stage; >= 8 rows without receivers end an item and are
        // skipped (every row an item carries is read from HBM)
        auto nd = [&](int64_t r) {
          return low.term_ptr[g.term_ptr + r + 1] - low.term_ptr[g.term_ptr + r];
        };
        auto& fr = franges[q - i];
        const int64_t max_rows = std::min<int64_t>(lim.max_rows, kMaxFoldRows);
        int64_t r = 0;
        while (r < g.n_rows) {
          while (r < g.n_rows && nd(r) == 0) ++r;
          if (r >= g.n_rows) break;
          const int64_t r0 = r;
          int64_t nt = 0, last = r;  // last row with receivers + 1
          while (r < g.n_rows) {
            const int64_t c = nd(r);
            if (c == 0 && r - last + 1 >= 8) break;
            const int64_t rows = r - r0 + 1;
            if (rows > 1 && (rows > max_rows || nt + c > kMaxItemTerms ||
                             rows * row16 + ((nt + c) * 4 + 15) / 16 * 16 + 16 > cap))
              break;
            nt += c;
            ++r;
            if (c) last = r;
          }
          fr.push_back({r0, last});
          r = last;
        }
        b.assign(fr.size() + 1, 0);
      } else if (g.op != OP_FOLD && g.op != OP_COPY) {
        b.push_back(0);  // READY / WAIT: one empty item
      }
      max_chunks = std::max(max_chunks, b.size() - 1);
    }
    // interleave the chunks of the groups of this stage (all peers / sources busy at once); with
    // lim.owner_major the forward COPY groups of one executing rank (one owner's embeddings to
    // each of its receivers, adjacent in [i, j)) are interleaved among themselves and the ranks
    // follow each other: the launch's write front is a few long runs of halo rows instead of one
    // chunk of every (owner, receiver) pair, and the owner's rows stay in L2 for its receivers
    std::vector<std::pair<size_t, size_t>> spans;  // [qb, qe) interleaved together
    for (size_t qb = i; qb < j;) {
      size_t qe = qb + 1;
      const DevGroup &gb = low.groups[gids[qb]];
      const bool om = lim.owner_major && gb.op == OP_COPY && gb.dir == DIR_FWD;
      // (owner_major 2: every forward COPY group on its own — one write run at a time)
      while (qe < j && (!om || (lim.owner_major == 1 &&
                                low.groups[gids[qe]].exec_rank == gb.exec_rank &&
                                low.groups[gids[qe]].op == OP_COPY)))
        ++qe;
      spans.push_back({qb, qe});
      qb = qe;
    }
    for (const auto &sp : spans)
    for (size_t c = 0; c < max_chunks; ++c) {
      for (size_t q = sp.first; q < sp.second; ++q) {
        const DevGroup &g = low.groups[gids[q]];
        const std::vector<int32_t> &b = bounds[q - i];
        if (c + 1 >= b.size()) continue;
        const bool fan = g.op == OP_FANOUT;
        const bool data = g.op == OP_COPY || g.op == OP_FOLD || fan;
        if (data && !fan && b[c + 1] == b[c]) continue;  // (empty chunk of a source-aligned set)
        const int64_t rb = fan ? franges[q - i][c].first : b[c];
        DevItem it;
        std::memset(&it, 0, sizeof(it));
        it.op = (uint8_t)g.op;
        it.dir = (uint8_t)g.dir;
        it.exec_rank = (uint8_t)g.exec_rank;
        it.dst_rank = (uint8_t)g.dst_rank;
        it.src_kind = (uint8_t)g.src_kind;
        it.dst_kind = (uint8_t)g.dst_kind;
        it.fold_init = (uint8_t)g.fold_init;
        it.term_mode = (uint8_t)g.term_mode;
        it.ready_rank = (int8_t)g.ready_rank;
        it.wait_n = (int16_t)g.wait_n;
        it.wait_off = g.wait_off;
        it.sig_ctr = g.sig_ctr;
        it.group = gids[q];
        it.rows = !data ? 0 : fan ? (int32_t)(franges[q - i][c].second - rb) : b[c + 1] - b[c];
        it.src = g.src_idx >= 0 ? ~(g.src_idx + rb) : g.src_base + rb;
        it.dst = g.dst_idx >= 0 ? ~(g.dst_idx + rb) : g.dst_base + rb;
        if (fan) {
          it.dst = 0;
          it.tp = g.term_ptr + rb;
          it.t0 = low.term_ptr[it.tp];
          it.nterms = (int32_t)(low.term_ptr[it.tp + it.rows] - it.t0);
        } else if (g.op == OP_FOLD) {
          it.tp = g.term_ptr + rb;
          it.t0 = low.term_ptr[it.tp];
          it.nterms = (int32_t)(low.term_ptr[it.tp + it.rows] - it.t0);
          if (staged[q - i]) stage_fold_item(low, g, &it, runs, sterms);
        } else if (g.op == OP_COPY) {
          // maximal runs of consecutive source and destination rows (one bulk copy each)
          it.tp = (int64_t)runs->size();
          auto srow = [&](int64_t i) {
            return g.src_idx >= 0 ? (int64_t)low.idx[g.src_idx + i] : g.src_base + i;
          };
          auto drow = [&](int64_t i) {
            return g.dst_idx >= 0 ? (int64_t)low.idx[g.dst_idx + i] : g.dst_base + i;
          };
          for (int64_t i = rb; i < rb + it.rows;) {
            int64_t j = i + 1;
            while (j < rb + it.rows && srow(j) == srow(j - 1) + 1 && drow(j) == drow(j - 1) + 1)
              ++j;
            runs->push_back({(int32_t)srow(i), (int32_t)drow(i), (int32_t)(j - i), (int32_t)(i - rb)});
            i = j;
          }
          it.nterms = (int32_t)((int64_t)runs->size() - it.tp);
        }
        bool sig = data && g.sig_ctr >= 0;
        if (sig && !signal_all && (fan || g.dst_kind == K_MCAST)) {
          sig = false;  // needed by some receiver of the owner's rows
          for (int d = 0; d < low.m; ++d)
            if (d != g.exec_rank && needed_ctr[(size_t)d * kCtrSpace + g.sig_ctr]) sig = true;
        } else if (sig && !signal_all) {
          sig = needed_ctr[(size_t)g.dst_rank * kCtrSpace + g.sig_ctr] != 0;
        }
        it.flags |= sig ? kItemSignal : 0;
        // optional: items whose runs average fewer than `direct_copy_rows` rows are gathered by
        // the consumers with plain loads instead of one bulk copy per run (0 = never; measured
        // slower than per-row bulk copies on the BASELINE graphs)
        if (g.atomic_add) it.flags |= kItemAtomic;
        if (g.op == OP_COPY && direct_copy_rows > 0 && !g.atomic_add && g.dst_kind != K_MCAST &&
            (int64_t)it.nterms * direct_copy_rows > (int64_t)it.rows)
          it.flags |= kItemDirect;
        // source rows in short runs (< 4 rows on average) of embeddings, halos (relay
        // forwarding), relay staging or halo gradients, rows that fit one tensor box: gather four
        // rows per TMA instruction instead of one bulk copy per run (used only when the launch
        // provides the kind's tensor map, see ExecParams::gather4_mask)
        // (a 4-row group must start 128-B aligned in shared memory: row16 % 32 == 0)
        else if (g.op == OP_COPY && lim.lsu_gather && g.dst_kind != K_MCAST && g.src_idx >= 0 &&
                 row16 <= kGather4MaxRowBytes && (int64_t)it.nterms * 4 > (int64_t)it.rows)
          it.flags |= kItemLsu;
        else if (g.op == OP_COPY && g.src_kind < kG4Kinds && g.src_idx >= 0 &&
                 row16 <= kGather4MaxRowBytes && row16 % 32 == 0 &&
                 (int64_t)it.nterms * 4 > (int64_t)it.rows)
          it.flags |= kItemGather4;
        items->push_back(it);
      }
    }
    i = j;
  }
}

}  // namespace dgcl

namespace dgcl {

// Relay forwards with the leaf split (see lower_plan): the forwarded rows form the critical
// chain stage 1 -> 2 -> ... -> K (stage k+1's forwarded items wait on stage k's), the leaves
// feed nothing.  Build order is stage-major, so stage k+1's forwarded items were claimed only
// after all of stage k's leaves, and then waited for the stage-k drain.  Here the chain goes
// first: after stage k's forwarded items come about `lead_bytes` of leaves (any stage <= k: all
// runnable by then) to cover the drain, then stage k+1's forwarded items; the remaining leaves
// last.  Every item still follows the items it waits on (deadlock-free in list order).
void lead_relay_items(const Lowered &low, std::vector<DevItem> *items, int64_t row_bytes,
                      int64_t lead_bytes) {
  if (low.leaf_block < 0 || lead_bytes < 0 || items->empty()) return;
  const int64_t row16 = (row_bytes + 15) / 16 * 16;
  std::vector<DevItem> head, tail;
  std::vector<std::vector<DevItem>> chain(kMaxStages + 1), leaves(kMaxStages + 1);
  int K = 0;
  for (const DevItem &it : *items) {
    if (it.op == OP_READY) {
      head.push_back(it);
      continue;
    }
    if (it.op == OP_WAIT) {
      tail.push_back(it);
      continue;
    }
    const DevGroup &g = low.groups[it.group];
    if (g.dir != DIR_FWD || g.stage < 1 || g.stage > kMaxStages) return;  // (not a relay forward)
    K = std::max(K, (int)g.stage);
    (g.block == low.leaf_block ? leaves : chain)[g.stage].push_back(it);
  }
  std::vector<DevItem> out = head;
  std::deque<DevItem> pool;
  for (int k = 1; k <= K; ++k) {
    out.insert(out.end(), chain[k].begin(), chain[k].end());
    pool.insert(pool.end(), leaves[k].begin(), leaves[k].end());
    bool more = false;  // forwarded rows in a later stage
    for (int j = k + 1; j <= K && !more; ++j) more = !chain[j].empty();
    if (!more) continue;
    int64_t b = 0;
    while (!pool.empty() && b < lead_bytes) {
      b += (int64_t)pool.front().rows * row16;
      out.push_back(pool.front());
      pool.pop_front();
    }
  }
  out.insert(out.end(), pool.begin(), pool.end());
  out.insert(out.end(), tail.begin(), tail.end());
  if (out.size() == items->size()) items->swap(out);
}

}  // namespace dgcl
