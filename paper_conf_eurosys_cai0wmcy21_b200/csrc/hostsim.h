// hostsim.h — host interpreter of lowered groups (verification aid, see hostsim.cpp).
#pragma once

#include <vector>

#include "plan.h"

namespace dgcl {

void hostsim_run(const Lowered &low, const std::vector<int32_t> &gids,
                 const std::vector<int64_t> &row_off, const std::vector<int64_t> &halo_off,
                 int64_t pitch, int dim, const float *emb, float *halo, const float *halo_grad,
                 float *emb_grad);

// the fused loopback program's work items, moved the way the bulk-copy executor moves them
// (row runs, staged FOLD segments + staged terms): checks build_items on the host; false if an
// item is malformed
bool hostsim_run_items(const Lowered &low, const std::vector<DevItem> &items,
                       const std::vector<DevRun> &runs, const std::vector<uint32_t> &sterms,
                       const std::vector<int64_t> &row_off, const std::vector<int64_t> &halo_off,
                       int64_t pitch, int dim, const float *emb, float *halo,
                       const float *halo_grad, float *emb_grad);

}  // namespace dgcl
