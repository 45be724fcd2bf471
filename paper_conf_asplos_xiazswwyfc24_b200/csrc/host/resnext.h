// Pattern lowering for the ResNeXt Bottleneck block (Table 2, ResNeXt-101 64 x 4d;
// SURVEY.md §8(f) NEXT-3): the TE program of models.resnext (1x1 convolutions as matmuls, the grouped 3x3
// convolution as rolled + border-masked taps with one batched matmul over the groups per tap, BatchNorm
// as a per-channel affine), fp32, one persistent launch (kernels/resnext.cu).  Ablation flags select
// the generic executor (the Table 4 ladder).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../resnext_types.h"
#include "ir.h"

namespace souffle {

struct RxPlan {
  bool on = false;
  std::string why_not;
  int x = -1, W1 = -1, s1 = -1, b1 = -1, s2 = -1, b2 = -1, W3 = -1, s3 = -1, b3 = -1, Wd = -1, sd = -1, bd = -1, y = -1;
  int W2[RX_TAPS], m[RX_TAPS];
  int H = 0, cin = 0, w = 0, G = 0, stride = 1, cout = 0, grid = 0, num_sp = 0;
  int64_t o_ctrl = 0, o_a = 0, o_d = 0, o_acc1 = 0, o_acc2 = 0, o_acc3 = 0, o_cnt = 0, total = 0;
};

void resnext_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, RxPlan& rp);
std::string resnext_describe(const RxPlan& rp);

}  // namespace souffle
