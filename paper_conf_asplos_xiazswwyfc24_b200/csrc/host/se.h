// Pattern lowering for the EfficientNet squeeze-and-excitation sub-module (Fig. 5 / 6;
// SURVEY.md §8(f) NEXT-3 M0-M9): y = x * sigmoid(fc2(silu(fc1(mean_rows(x))))), fp32, one
// subprogram -> one persistent launch (kernels/se.cu).  Flags 0: global sync + data reuse (Fig. 5(d));
// SOUFFLE_FLAG_NO_PREFETCH: global sync without the shared-memory reuse of x (Fig. 5(c)).
#pragma once
#include <cstdint>
#include <string>

#include "../se_types.h"
#include "ir.h"

namespace souffle {

struct SePlan {
  bool on = false;
  std::string why_not;
  int x = -1, W1 = -1, b1 = -1, W2 = -1, b2 = -1, y = -1;
  int HW = 0, C = 0, S = 0, nrb = 0, ncb = 0, rows = 0, cbw = 0, reuse = 1;
  int64_t o_part = 0, o_pooled = 0, o_h = 0, o_ctrl = 0, total = 0;
};

void se_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, SePlan& sp);
std::string se_describe(const SePlan& sp);

}  // namespace souffle
