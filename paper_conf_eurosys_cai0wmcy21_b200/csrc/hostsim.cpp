// hostsim.cpp — single-threaded host interpreter of the lowered groups (verification aid).
//
// Runs exactly the group descriptors and index pools the device executor consumes, in the same
// stage order and with the same fp32 fold order, on host buffers in the loopback layouts.  It lets
// the CPU test-suite check planning + lowering against the oracle without a GPU.  It is NOT a
// fallback: dgcl_dispatch_* never reaches it (see dgcl.h, "verification aids").

#include <cmath>
#include <cstring>
#include <vector>

#include "hostsim.h"

namespace dgcl {

namespace {

struct HostBufs {
  float *base[K_NKINDS][kMaxRanks];
  int64_t pitch;  // elements, same for every buffer
};

inline float *row_ptr(const HostBufs &B, int kind, int rank, int64_t row) {
  return B.base[kind][rank] + row * B.pitch;
}

// a row stored into destination (kind, rank, row): the multicast region kind reaches every
// rank's copy (what one store through the multicast address does)
inline void put_row(const HostBufs &B, int m, int kind, int rank, int64_t row, const float *s,
                    int dim) {
  if (kind == K_MCAST) {
    for (int r = 0; r < m; ++r) std::memcpy(row_ptr(B, K_MCUC, r, row), s, sizeof(float) * dim);
    return;
  }
  std::memcpy(row_ptr(B, kind, rank, row), s, sizeof(float) * dim);
}

// OP_FANOUT rows [r0, r0 + rows) of group g: each source row into all its receivers' rows
bool run_fanout(const Lowered &low, const DevGroup &g, int64_t r0, int64_t rows,
                const HostBufs &B, int dim) {
  for (int64_t r = r0; r < r0 + rows; ++r) {
    const float *s = row_ptr(B, g.src_kind, g.exec_rank, g.src_base + r);
    for (int64_t t = low.term_ptr[g.term_ptr + r]; t < low.term_ptr[g.term_ptr + r + 1]; t += 2) {
      const uint32_t d = low.terms[t];
      if ((int64_t)low.terms[t + 1] != g.src_base + r) return false;  // (source row of the pair)
      std::memcpy(row_ptr(B, (d & kFanRelay) ? K_RELAY : K_HALO, (int)(d >> 28), d & kFanRowMask),
                  s, sizeof(float) * dim);
    }
  }
  return true;
}

// kTermRankTree postfix program: each word pushes its operand, then (word >> 24) & 15 adds of
// the top two (below + top); the stack bottom is the starting value
template <typename Val>
float eval_tree(float init, const uint32_t *prog, int64_t n, Val val) {
  std::vector<float> stk(1, init);
  for (int64_t j = 0; j < n; ++j) {
    stk.push_back(val(prog[j]));
    for (uint32_t a = (prog[j] >> kTreeAddShift) & 15u; a > 0; --a) {
      if (stk.size() < 2) return std::nanf("");  // (malformed program poisons the row)
      volatile float t = stk.back();
      stk.pop_back();
      stk.back() = stk.back() + t;
    }
  }
  return stk.size() == 1 ? stk[0] : std::nanf("");
}

void run_group(const Lowered &low, const DevGroup &g, const HostBufs &B, int dim) {
  if (g.op == OP_READY || g.op == OP_WAIT) return;
  if (g.op == OP_FANOUT) {
    run_fanout(low, g, 0, g.n_rows, B, dim);
    return;
  }
  for (int64_t i = 0; i < g.n_rows; ++i) {
    const int64_t drow = g.dst_idx >= 0 ? low.idx[g.dst_idx + i] : g.dst_base + i;
    float *d = g.dst_kind == K_MCAST ? nullptr : row_ptr(B, g.dst_kind, g.dst_rank, drow);
    if (g.op == OP_COPY) {
      const int64_t srow = g.src_idx >= 0 ? low.idx[g.src_idx + i] : g.src_base + i;
      const float *s = row_ptr(B, g.src_kind, g.exec_rank, srow);
      if (g.atomic_add)
        for (int c = 0; c < dim; ++c) d[c] += s[c];
      else
        put_row(B, low.m, g.dst_kind, g.dst_rank, drow, s, dim);
    } else {
      const int64_t t0 = low.term_ptr[g.term_ptr + i], t1 = low.term_ptr[g.term_ptr + i + 1];
      auto operand = [&](uint32_t term) -> const float * {
        if (g.term_mode == kTermRankHgrad)
          return row_ptr(B, K_HGRAD, (int)(term >> 28), term & kTermRowMask);
        return row_ptr(B, (term & kTermSlot) ? K_SLOT : K_HGRAD, g.exec_rank, term & ~kTermSlot);
      };
      if (g.term_mode == kTermRankTree) {
        for (int c = 0; c < dim; ++c)
          d[c] = eval_tree(d[c], low.terms.data() + t0, t1 - t0, [&](uint32_t w) {
            return row_ptr(B, K_HGRAD, (int)(w >> 28), w & kTreeRowMask)[c];
          });
        continue;
      }
      for (int c = 0; c < dim; ++c) {
        int64_t t = t0;
        float acc;
        if (g.fold_init)
          acc = d[c];
        else
          acc = operand(low.terms[t++])[c];
        for (; t < t1; ++t) {
          volatile float v = operand(low.terms[t])[c];
          acc = acc + v;  // one IEEE fp32 add per term, in list order
        }
        d[c] = acc;
      }
    }
  }
}

// one work item the way the bulk-copy executor moves it: COPY items by their row runs, staged
// FOLD items through an emulated shared-memory stage (segments copied in, terms read back by
// their staged rows), other FOLD items term by term
// returns false if the item is malformed (shape checks the device executor relies on)
bool run_item(const Lowered &low, const DevItem &it, const std::vector<DevRun> &runs,
              const std::vector<uint32_t> &sterms, const HostBufs &B, int dim) {
  if (it.op != OP_COPY && it.op != OP_FOLD && it.op != OP_FANOUT) return it.rows == 0;
  if (it.rows <= 0 || it.rows > (it.op == OP_COPY ? kMaxItemRows : kMaxFoldRows)) return false;
  if (it.op == OP_FANOUT) {
    const DevGroup &g = low.groups[it.group];
    const int64_t r0 = it.src - g.src_base;
    if (it.tp != g.term_ptr + r0 || it.t0 != low.term_ptr[it.tp] ||
        it.nterms != low.term_ptr[it.tp + it.rows] - it.t0 || it.nterms < 1 ||
        it.nterms > kMaxItemTerms)
      return false;
    return run_fanout(low, g, r0, it.rows, B, dim);
  }
  auto drow = [&](int64_t r) { return it.dst >= 0 ? it.dst + r : (int64_t)low.idx[~it.dst + r]; };
  if (it.op == OP_COPY) {
    int64_t covered = 0;
    for (int32_t q = 0; q < it.nterms; ++q) {
      const DevRun &R = runs[it.tp + q];
      if (R.pos != covered || R.len < 1) return false;
      covered += R.len;
      for (int32_t j = 0; j < R.len; ++j) {
        const float *s = row_ptr(B, it.src_kind, it.exec_rank, R.src + j);
        if (it.flags & kItemAtomic) {
          float *d = row_ptr(B, it.dst_kind, it.dst_rank, R.dst + j);
          for (int c = 0; c < dim; ++c) d[c] += s[c];
        } else {
          put_row(B, low.m, it.dst_kind, it.dst_rank, R.dst + j, s, dim);
        }
      }
    }
    return covered == it.rows;
  }
  const int64_t *tp = low.term_ptr.data() + it.tp;
  if (it.flags & kItemStaged) {
    const int64_t nseg = it.src >> kSegShift, seg0 = it.src & ((1ll << kSegShift) - 1);
    const int64_t nst = (it.fold_init ? it.rows : 0) + it.nterms;  // stage rows reserved
    if (nst > kMaxItemRows || nseg < 1 || nseg > nst) return false;
    std::vector<float> stage((size_t)nst * B.pitch, std::nanf(""));
    std::vector<uint8_t> hit(nst, 0);
    for (int64_t q = 0; q < nseg; ++q) {
      const DevRun &R = runs[seg0 + q];
      if (R.pos < 0 || R.len < 1 || R.pos + R.len > nst) return false;
      for (int32_t j = 0; j < R.len; ++j) {
        if (hit[R.pos + j]) return false;
        hit[R.pos + j] = 1;
      }
      for (int32_t j = 0; j < R.len; ++j)
        std::memcpy(&stage[(size_t)(R.pos + j) * B.pitch],
                    row_ptr(B, R.dst >> 8, R.dst & 255, R.src + j), sizeof(float) * dim);
    }
    for (int64_t r = 0; r < it.rows; ++r) {
      float *d = row_ptr(B, it.dst_kind, it.dst_rank, drow(r));
      if (low.groups[it.group].term_mode == kTermRankTree) {
        const int64_t j = tp[r] - tp[0], je = tp[r + 1] - tp[0];
        for (int c = 0; c < dim; ++c)
          d[c] = eval_tree(stage[(size_t)r * B.pitch + c], sterms.data() + it.t0 + j, je - j,
                           [&](uint32_t s) { return stage[(size_t)(s & kTreeRowMask) * B.pitch + c]; });
        continue;
      }
      for (int c = 0; c < dim; ++c) {
        int64_t j = tp[r] - tp[0];
        const int64_t je = tp[r + 1] - tp[0];
        float acc = it.fold_init ? stage[(size_t)r * B.pitch + c]
                                 : stage[(size_t)sterms[it.t0 + j++] * B.pitch + c];
        for (; j < je; ++j) {
          volatile float v = stage[(size_t)sterms[it.t0 + j] * B.pitch + c];
          acc = acc + v;
        }
        d[c] = acc;
      }
    }
    for (uint8_t h : hit)
      if (!h) return false;  // every staged row is filled by exactly one segment
    return true;
  }
  DevGroup g = low.groups[it.group];
  g.n_rows = it.rows;
  g.term_ptr = it.tp;
  g.dst_idx = it.dst < 0 ? ~it.dst : -1;
  g.dst_base = it.dst;
  run_group(low, g, B, dim);
  return true;
}

void setup_bufs(const Lowered &low, const std::vector<int64_t> &row_off,
                const std::vector<int64_t> &halo_off, int64_t pitch, const float *emb, float *halo,
                const float *halo_grad, float *emb_grad, std::vector<std::vector<float>> &relay,
                std::vector<std::vector<float>> &slot, HostBufs *B) {
  const int m = low.m;
  relay.assign(m, {});
  slot.assign(m, {});
  // (the multicast region copies live after the relay / slot buffers of `relay`)
  relay.resize(2 * m);
  std::memset(B, 0, sizeof(*B));
  B->pitch = pitch;
  for (int r = 0; r < m; ++r) {
    relay[r].assign((size_t)low.n_relay[r] * pitch, 0.f);
    slot[r].assign((size_t)low.n_slot[r] * pitch, 0.f);
    B->base[K_EMB][r] = const_cast<float *>(emb) + (emb ? row_off[r] * pitch : 0);
    B->base[K_EGRAD][r] = emb_grad + (emb_grad ? row_off[r] * pitch : 0);
    B->base[K_HALO][r] = halo + (halo ? halo_off[r] * pitch : 0);
    B->base[K_HGRAD][r] = const_cast<float *>(halo_grad) + (halo_grad ? halo_off[r] * pitch : 0);
    B->base[K_RELAY][r] = relay[r].data();
    B->base[K_SLOT][r] = slot[r].data();
    relay[m + r].assign((size_t)low.mc_total * pitch, 0.f);
    B->base[K_MCUC][r] = relay[m + r].data();
  }
}

}  // namespace

bool hostsim_run_items(const Lowered &low, const std::vector<DevItem> &items,
                       const std::vector<DevRun> &runs, const std::vector<uint32_t> &sterms,
                       const std::vector<int64_t> &row_off, const std::vector<int64_t> &halo_off,
                       int64_t pitch, int dim, const float *emb, float *halo,
                       const float *halo_grad, float *emb_grad) {
  std::vector<std::vector<float>> relay, slot;
  HostBufs B;
  setup_bufs(low, row_off, halo_off, pitch, emb, halo, halo_grad, emb_grad, relay, slot, &B);
  for (const DevItem &it : items)  // stage order
    if (!run_item(low, it, runs, sterms, B, dim)) return false;
  return true;
}

void hostsim_run(const Lowered &low, const std::vector<int32_t> &gids,
                 const std::vector<int64_t> &row_off, const std::vector<int64_t> &halo_off,
                 int64_t pitch, int dim, const float *emb, float *halo, const float *halo_grad,
                 float *emb_grad) {
  std::vector<std::vector<float>> relay, slot;
  HostBufs B;
  setup_bufs(low, row_off, halo_off, pitch, emb, halo, halo_grad, emb_grad, relay, slot, &B);
  for (int32_t gi : gids) {  // the program's groups, in stage order
    const DevGroup &g = low.groups[gi];
    if (g.op == OP_READY || g.op == OP_WAIT) continue;
    run_group(low, g, B, dim);
  }
}

}  // namespace dgcl
