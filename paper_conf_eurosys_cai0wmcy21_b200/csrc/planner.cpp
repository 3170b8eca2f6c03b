// planner.cpp — communication relation and the SPST planner (host only, no CUDA).
//
// PAPER.md §5.  The planning problem (eq. 2) is: choose for every vertex
// u a tree T_u rooted at its owner s_u spanning the requesting GPUs D_u, minimising the staged
// cost t(S) of §5.1.  SPST (Algorithm 1) plans vertices one by one in a random order;
// per vertex it repeatedly runs a multi-source Dijkstra from the GPUs already holding u (N_src) to
// the unreached requesters, with edge weights from incrementalLinkCost (Algorithm 2):
// C(i, e) = costFunc(S + {(i, e)}) - costFunc(S), and adds the cheapest path.
//
// Readings (R7-R12): integer ticks per row per hop; node-labelled Dijkstra where x->y
// weighs C(depth(x)+1, x->y); labels compare (cost, depth, gpu id); target = min (cost, depth, id);
// stop once D_u is covered; Fisher-Yates shuffle driven by splitmix64(seed).  C is evaluated on
// demand for the relaxed edges only (the optimisation the paper mentions at P:1384-1392): because
// S is fixed during one Dijkstra, C(k, e) = max(t^k, max_{h in e} (c_h^k + 1) w_h) - t^k exactly.

#include <algorithm>
#include <chrono>
#include <cstring>
#include <string>

#include "plan.h"

namespace dgcl {

Topology Topology::uniform_nvswitch(int m) {
  // link i->j = {egress_i, ingress_j}; 900 GB/s each => round(1e5 / 900) = 111 ticks per row
  Topology t;
  t.m = m;
  t.w.assign(2 * m, 111);
  t.link_ptr.assign((size_t)m * m + 1, 0);
  for (int i = 0; i < m; ++i)
    for (int j = 0; j < m; ++j) {
      size_t p = (size_t)i * m + j;
      if (i != j) {
        t.link_hops.push_back(i);
        t.link_hops.push_back(m + j);
      }
      t.link_ptr[p + 1] = (int64_t)t.link_hops.size();
    }
  return t;
}

std::string build_relation(int64_t n, int m, const int32_t *part, const int64_t *req_ptr,
                           const int64_t *req_ids, Relation *out) {
  Relation &r = *out;
  r.n = n;
  r.m = m;
  r.n_halo.assign(m, 0);
  if (req_ptr[0] != 0) return "req_ptr[0] must be 0";
  for (int d = 0; d < m; ++d) {
    if (req_ptr[d + 1] < req_ptr[d]) return "req_ptr must be non-decreasing";
    r.n_halo[d] = req_ptr[d + 1] - req_ptr[d];
  }
  const int64_t S = req_ptr[m];
  std::vector<int64_t> cnt(n + 1, 0);
  for (int d = 0; d < m; ++d) {
    for (int64_t i = req_ptr[d]; i < req_ptr[d + 1]; ++i) {
      const int64_t u = req_ids[i];
      if (u < 0 || u >= n) return "required id out of range: " + std::to_string(u);
      if (part[u] == d)
        return "GPU " + std::to_string(d) + " requires its own vertex " + std::to_string(u);
      cnt[u + 1]++;
    }
  }
  r.d_ptr.assign(n + 1, 0);
  for (int64_t u = 0; u < n; ++u) r.d_ptr[u + 1] = r.d_ptr[u] + cnt[u + 1];
  r.d_gpu.assign(S, -1);
  r.d_pos.assign(S, -1);
  std::vector<int64_t> fill(r.d_ptr.begin(), r.d_ptr.end() - 1);
  for (int d = 0; d < m; ++d) {  // ascending d => each D_u list is sorted
    for (int64_t i = req_ptr[d]; i < req_ptr[d + 1]; ++i) {
      const int64_t u = req_ids[i];
      const int64_t f = fill[u];
      if (f > r.d_ptr[u] && r.d_gpu[f - 1] == d)
        return "duplicate id " + std::to_string(u) + " in the list of GPU " + std::to_string(d);
      r.d_gpu[f] = (int8_t)d;
      r.d_pos[f] = (int32_t)(i - req_ptr[d]);
      fill[u] = f + 1;
    }
  }
  return "";
}

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;
inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

constexpr int64_t kInf = INT64_MAX;

// Is the topology the uniform switch model (link i->j = {egress_i, ingress_j}, every hop the same
// cost, egress and ingress hops all distinct)?  Then SPST provably plans every delivery directly
// in stage 1, in any vertex order: stage 2 carries no load (induction), so any 2-hop path costs at
// least C(2, .) = w, while a direct link costs C(1, s->d) = max((c+1) w) - t^1 <= w (t^1 >= c w for
// every stage-1 hop) and wins ties on depth (R8); the trees are stars, t(S) = w x the largest
// egress / ingress row count.  (the closed form behind the parallel planner.)
bool uniform_switch(const Topology &t) {
  const int m = t.m;
  if (m < 2 || t.w.empty()) return false;
  std::vector<int32_t> eg(m, -1), ig(m, -1);
  for (int i = 0; i < m; ++i)
    for (int j = 0; j < m; ++j) {
      if (i == j) continue;
      const int64_t a = t.link_ptr[(size_t)i * m + j], b = t.link_ptr[(size_t)i * m + j + 1];
      if (b - a != 2) return false;
      const int32_t h0 = t.link_hops[a], h1 = t.link_hops[a + 1];
      if (t.w[h0] != t.w[0] || t.w[h1] != t.w[0] || h0 == h1) return false;
      if ((eg[i] >= 0 && eg[i] != h0) || (ig[j] >= 0 && ig[j] != h1)) return false;
      eg[i] = h0;
      ig[j] = h1;
    }
  std::vector<int32_t> all(eg);
  all.insert(all.end(), ig.begin(), ig.end());
  std::sort(all.begin(), all.end());
  return std::adjacent_find(all.begin(), all.end()) == all.end();
}

}  // namespace

std::string spst_plan(const Topology &topo, const int32_t *part, const Relation &rel,
                      uint64_t seed, Plan *out, bool allow_fast) {
  auto t0 = std::chrono::steady_clock::now();
  const int m = topo.m;
  Plan &P = *out;
  P = Plan();
  P.m = m;
  // vertices with D_u non-empty, ascending, then Fisher-Yates (splitmix64 stream from `seed`)
  std::vector<int64_t> &order = P.order;
  for (int64_t u = 0; u < rel.n; ++u)
    if (rel.d_ptr[u + 1] > rel.d_ptr[u]) order.push_back(u);
  {
    uint64_t state = seed;
    for (int64_t i = (int64_t)order.size() - 1; i >= 1; --i) {
      state += kGolden;
      const int64_t j = (int64_t)(mix64(state) % (uint64_t)(i + 1));
      std::swap(order[i], order[j]);
    }
  }
  const int H = (int)topo.w.size();
  if (allow_fast && uniform_switch(topo)) {
    // the closed form of SPST on the uniform switch (above): every vertex's tree is the star
    // owner -> each requester (ascending id: the canonical edge order), built in parallel
    const int64_t NV = (int64_t)order.size();
    P.e_ptr.assign(NV + 1, 0);
    for (int64_t i = 0; i < NV; ++i)
      P.e_ptr[i + 1] = P.e_ptr[i] + (rel.d_ptr[order[i] + 1] - rel.d_ptr[order[i]]);
    const int64_t NE = P.e_ptr[NV];
    P.e_parent.assign(NE, 0);
    P.e_child.assign(NE, 0);
    P.e_stage.assign(NE, 1);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < NV; ++i) {
      const int64_t u = order[i];
      int64_t e = P.e_ptr[i];
      for (int64_t q = rel.d_ptr[u]; q < rel.d_ptr[u + 1]; ++q, ++e) {
        P.e_parent[e] = part[u];
        P.e_child[e] = rel.d_gpu[q];
      }
    }
    std::vector<int64_t> out_rows(m, 0), in_rows(m, 0);
    for (int64_t u = 0; u < rel.n; ++u)
      for (int64_t q = rel.d_ptr[u]; q < rel.d_ptr[u + 1]; ++q) {
        ++out_rows[part[u]];
        ++in_rows[rel.d_gpu[q]];
      }
    int64_t mx = 0;
    for (int d = 0; d < m; ++d) mx = std::max(mx, std::max(out_rows[d], in_rows[d]));
    P.n_stages = NE > 0 ? 1 : 0;
    P.cost = mx * topo.w[0];
    P.closed_form = true;
    P.seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    return "";
  }
  // c_h^k and t^k, k in 1..m-1 (row 0 unused)
  std::vector<int64_t> load((size_t)m * H, 0);
  std::vector<int64_t> tk(m, 0);
  const int64_t S = rel.d_ptr[rel.n];
  P.e_ptr.reserve(order.size() + 1);
  P.e_parent.reserve(S);
  P.e_child.reserve(S);
  P.e_stage.reserve(S);
  P.e_ptr.push_back(0);

  // per-link hop lists as small arrays
  std::vector<int32_t> lp(topo.link_ptr.begin(), topo.link_ptr.end());

  auto inc_cost = [&](int k, int x, int y) -> int64_t {
    // C(k, x->y) = costFunc(S + {(k, x->y)}) - costFunc(S): only stage k changes
    const int64_t cur = tk[k];
    int64_t mx = cur;
    const int64_t *ld = &load[(size_t)k * H];
    for (int32_t q = lp[x * m + y]; q < lp[x * m + y + 1]; ++q) {
      const int h = topo.link_hops[q];
      const int64_t v = (ld[h] + 1) * topo.w[h];
      if (v > mx) mx = v;
    }
    return mx - cur;
  };

  int max_stage = 0;
  int64_t lcost[kMaxRanks];
  int ldep[kMaxRanks], pred[kMaxRanks], depth[kMaxRanks];
  for (const int64_t u : order) {
    const int su = part[u];
    uint32_t in_src = 1u << su;
    for (int x = 0; x < m; ++x) depth[x] = -1;
    depth[su] = 0;
    uint32_t remaining = 0;
    for (int64_t q = rel.d_ptr[u]; q < rel.d_ptr[u + 1]; ++q) remaining |= 1u << rel.d_gpu[q];
    while (remaining) {
      // --- multi-source node-labelled Dijkstra (Algorithm 1 line 7) ---
      for (int x = 0; x < m; ++x) {
        if (in_src >> x & 1) {
          lcost[x] = 0;
          ldep[x] = depth[x];
        } else {
          lcost[x] = kInf;
          ldep[x] = INT32_MAX;
        }
        pred[x] = -1;
      }
      uint32_t settled = 0;
      for (;;) {
        int bx = -1;
        for (int x = 0; x < m; ++x) {
          if ((settled >> x & 1) || lcost[x] == kInf) continue;
          if (bx < 0 || lcost[x] < lcost[bx] || (lcost[x] == lcost[bx] && ldep[x] < ldep[bx]))
            bx = x;  // ascending x breaks the remaining ties
        }
        if (bx < 0) break;
        settled |= 1u << bx;
        const int k = ldep[bx] + 1;
        if (k > m - 1) continue;
        for (int y = 0; y < m; ++y) {
          if (y == bx || (settled >> y & 1) || (in_src >> y & 1) || !topo.has(bx, y)) continue;
          const int64_t c = lcost[bx] + inc_cost(k, bx, y);
          if (c < lcost[y] || (c == lcost[y] && k < ldep[y])) {
            lcost[y] = c;
            ldep[y] = k;
            pred[y] = bx;
          }
        }
      }
      // --- Algorithm 1 line 8: cheapest path to an unreached requester ---
      int tgt = -1;
      for (int d = 0; d < m; ++d) {
        if (!(remaining >> d & 1) || lcost[d] == kInf) continue;
        if (tgt < 0 || lcost[d] < lcost[tgt] || (lcost[d] == lcost[tgt] && ldep[d] < ldep[tgt]))
          tgt = d;
      }
      if (tgt < 0)
        return "vertex " + std::to_string(u) + ": a requesting GPU is unreachable from GPU " +
               std::to_string(su);
      // walk back to N_src, then add nodes and edges (lines 9-10) in root-to-leaf order
      int path[kMaxRanks];
      int np = 0;
      for (int y = tgt; !(in_src >> y & 1); y = pred[y]) path[np++] = y;
      for (int i = np - 1; i >= 0; --i) {
        const int c = path[i];
        const int p = pred[c];
        const int k = depth[p] + 1;
        depth[c] = k;
        in_src |= 1u << c;
        remaining &= ~(1u << c);
        P.e_parent.push_back(p);
        P.e_child.push_back(c);
        P.e_stage.push_back(k);
        if (k > max_stage) max_stage = k;
        int64_t *ld = &load[(size_t)k * H];
        for (int32_t q = lp[p * m + c]; q < lp[p * m + c + 1]; ++q) {
          const int h = topo.link_hops[q];
          ld[h] += 1;
          const int64_t v = ld[h] * topo.w[h];
          if (v > tk[k]) tk[k] = v;
        }
      }
    }
    // canonical edge order within T_u: (stage, child) — a tree is a set of edges; this order
    // keeps parents before children (R26)
    {
      const int64_t b = P.e_ptr.back(), e = (int64_t)P.e_parent.size();
      int64_t idx[kMaxRanks];
      int32_t pp[kMaxRanks], cc[kMaxRanks], kk[kMaxRanks];
      const int n = (int)(e - b);
      for (int i = 0; i < n; ++i) idx[i] = b + i;
      std::sort(idx, idx + n, [&](int64_t x, int64_t y) {
        return P.e_stage[x] != P.e_stage[y] ? P.e_stage[x] < P.e_stage[y]
                                            : P.e_child[x] < P.e_child[y];
      });
      for (int i = 0; i < n; ++i) {
        pp[i] = P.e_parent[idx[i]];
        cc[i] = P.e_child[idx[i]];
        kk[i] = P.e_stage[idx[i]];
      }
      for (int i = 0; i < n; ++i) {
        P.e_parent[b + i] = pp[i];
        P.e_child[b + i] = cc[i];
        P.e_stage[b + i] = kk[i];
      }
    }
    P.e_ptr.push_back((int64_t)P.e_parent.size());
  }
  P.n_stages = max_stage;
  P.cost = 0;
  for (int k = 1; k < m; ++k) P.cost += tk[k];
  P.seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  return "";
}

// A plan given as trees (e.g. saved from dgcl_plan_export of an earlier run: planning happens
// once before training, and costs seconds to minutes at scale, Table 8):
// edges grouped per vertex, each group in root-to-leaf order (a parent is the owner or an
// earlier child).  Checks the §8(c) plan invariants and recomputes t(S) with the §5.1 rules.
std::string import_plan(const Topology &topo, const int32_t *part, const Relation &rel,
                        int64_t n_edges, const int64_t *u, const int32_t *parent,
                        const int32_t *child, const int32_t *stage, Plan *out) {
  Plan &P = *out;
  P = Plan();
  const int m = topo.m;
  P.m = m;
  const int H = (int)topo.w.size();
  std::vector<int64_t> load((size_t)kMaxStages * H, 0);
  std::vector<int64_t> tk(kMaxStages, 0);
  std::vector<uint8_t> seen(rel.n, 0);
  int64_t planned = 0;
  for (int64_t v = 0; v < rel.n; ++v) planned += rel.d_ptr[v + 1] > rel.d_ptr[v] ? 1 : 0;
  P.e_ptr.push_back(0);
  int max_stage = 0;
  for (int64_t e = 0; e < n_edges;) {
    const int64_t v = u[e];
    if (v < 0 || v >= rel.n) return "edge " + std::to_string(e) + ": vertex out of range";
    if (seen[v]) return "vertex " + std::to_string(v) + ": its edges are not contiguous";
    seen[v] = 1;
    if (rel.d_ptr[v + 1] == rel.d_ptr[v])
      return "vertex " + std::to_string(v) + ": no GPU requests it";
    const int root = part[v];
    int depth[kMaxRanks], nchild[kMaxRanks];
    for (int x = 0; x < m; ++x) depth[x] = -1, nchild[x] = 0;
    depth[root] = 0;
    int64_t f = e;
    for (; f < n_edges && u[f] == v; ++f) {
      const int p = parent[f], c = child[f], k = stage[f];
      if (p < 0 || p >= m || c < 0 || c >= m) return "edge " + std::to_string(f) + ": GPU id";
      if (depth[p] < 0) return "edge " + std::to_string(f) + ": parent not yet in the tree";
      if (depth[c] >= 0) return "edge " + std::to_string(f) + ": node already in the tree";
      if (k != depth[p] + 1 || k > m - 1 || k >= kMaxStages)
        return "edge " + std::to_string(f) + ": stage is not the tree depth";
      if (!topo.has(p, c)) return "edge " + std::to_string(f) + ": no such link";
      depth[c] = k;
      nchild[p]++;
      max_stage = std::max(max_stage, k);
      P.e_parent.push_back(p);
      P.e_child.push_back(c);
      P.e_stage.push_back(k);
      int64_t *ld = &load[(size_t)k * H];
      for (int32_t q = topo.link_ptr[p * m + c]; q < topo.link_ptr[p * m + c + 1]; ++q) {
        const int h = topo.link_hops[q];
        ld[h] += 1;
        tk[k] = std::max(tk[k], ld[h] * topo.w[h]);
      }
    }
    uint32_t req = 0;
    for (int64_t q = rel.d_ptr[v]; q < rel.d_ptr[v + 1]; ++q) {
      req |= 1u << rel.d_gpu[q];
      if (depth[rel.d_gpu[q]] < 0)
        return "vertex " + std::to_string(v) + ": GPU " + std::to_string(rel.d_gpu[q]) +
               " requests it but is not in its tree";
    }
    for (int x = 0; x < m; ++x)  // a relay that forwards nothing would only waste a row
      if (x != root && depth[x] >= 0 && !(req >> x & 1) && nchild[x] == 0)
        return "vertex " + std::to_string(v) + ": GPU " + std::to_string(x) +
               " is a leaf that did not request it";
    P.order.push_back(v);
    P.e_ptr.push_back((int64_t)P.e_parent.size());
    e = f;
  }
  if ((int64_t)P.order.size() != planned)
    return "plan covers " + std::to_string(P.order.size()) + " of " + std::to_string(planned) +
           " requested vertices";
  P.n_stages = max_stage;
  P.cost = 0;
  for (int k = 1; k < kMaxStages; ++k) P.cost += tk[k];
  return "";
}

}  // namespace dgcl
