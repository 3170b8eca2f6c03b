// hostsim.cpp — single-threaded host interpreter of the lowered groups (verification aid).
//
// Runs exactly the group descriptors and index pools the device executor consumes, in the same
// stage order and with the same fp32 fold order, on host buffers in the loopback layouts.  It lets
// the CPU test-suite check planning + lowering against the oracle without a GPU.  It is NOT a
// fallback: dgcl_dispatch_* never reaches it (see dgcl.h, "verification aids").

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

void run_group(const Lowered &low, const DevGroup &g, const HostBufs &B, int dim) {
  if (g.op == OP_READY || g.op == OP_WAIT) return;
  for (int64_t i = 0; i < g.n_rows; ++i) {
    const int64_t drow = g.dst_idx >= 0 ? low.idx[g.dst_idx + i] : g.dst_base + i;
    float *d = row_ptr(B, g.dst_kind, g.dst_rank, drow);
    if (g.op == OP_COPY) {
      const int64_t srow = g.src_idx >= 0 ? low.idx[g.src_idx + i] : g.src_base + i;
      const float *s = row_ptr(B, g.src_kind, g.exec_rank, srow);
      std::memcpy(d, s, sizeof(float) * dim);
    } else {
      const int64_t t0 = low.term_ptr[g.term_ptr + i], t1 = low.term_ptr[g.term_ptr + i + 1];
      auto operand = [&](uint32_t term) -> const float * {
        if (g.term_mode == kTermRankHgrad)
          return row_ptr(B, K_HGRAD, (int)(term >> 28), term & kTermRowMask);
        return row_ptr(B, (term & kTermSlot) ? K_SLOT : K_HGRAD, g.exec_rank, term & ~kTermSlot);
      };
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

}  // namespace

void hostsim_run(const Lowered &low, const std::vector<int32_t> &gids,
                 const std::vector<int64_t> &row_off, const std::vector<int64_t> &halo_off,
                 int64_t pitch, int dim, const float *emb, float *halo, const float *halo_grad,
                 float *emb_grad) {
  const int m = low.m;
  std::vector<std::vector<float>> relay(m), slot(m);
  HostBufs B;
  std::memset(&B, 0, sizeof(B));
  B.pitch = pitch;
  for (int r = 0; r < m; ++r) {
    relay[r].assign((size_t)low.n_relay[r] * pitch, 0.f);
    slot[r].assign((size_t)low.n_slot[r] * pitch, 0.f);
    B.base[K_EMB][r] = const_cast<float *>(emb) + (emb ? row_off[r] * pitch : 0);
    B.base[K_EGRAD][r] = emb_grad + (emb_grad ? row_off[r] * pitch : 0);
    B.base[K_HALO][r] = halo + (halo ? halo_off[r] * pitch : 0);
    B.base[K_HGRAD][r] = const_cast<float *>(halo_grad) + (halo_grad ? halo_off[r] * pitch : 0);
    B.base[K_RELAY][r] = relay[r].data();
    B.base[K_SLOT][r] = slot[r].data();
  }
  for (int32_t gi : gids) {  // the program's groups, in stage order
    const DevGroup &g = low.groups[gi];
    if (g.op == OP_READY || g.op == OP_WAIT) continue;
    run_group(low, g, B, dim);
  }
}

}  // namespace dgcl
