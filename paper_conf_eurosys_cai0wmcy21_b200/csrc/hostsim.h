// hostsim.h — host interpreter of lowered groups (verification aid, see hostsim.cpp).
#pragma once

#include <vector>

#include "plan.h"

namespace dgcl {

void hostsim_run(const Lowered &low, const std::vector<int32_t> &gids,
                 const std::vector<int64_t> &row_off, const std::vector<int64_t> &halo_off,
                 int64_t pitch, int dim, const float *emb, float *halo, const float *halo_grad,
                 float *emb_grad);

}  // namespace dgcl
