// Pattern lowering for the EfficientNet MBConv block (Fig. 5 / 6, L1511-1564; SURVEY.md §8(f)
// NEXT-3): the TE program of models.mbconv (1x1 convolutions as matmuls, the depthwise convolution as
// rolled + border-masked taps, SE, BatchNorm as a per-channel affine), fp32, one persistent launch
// (kernels/mbconv.cu).  Flags 0: data reuse where it fits (Fig. 5(d)); SOUFFLE_FLAG_NO_PREFETCH: global
// sync with d through L2 (Fig. 5(c)); other flags select the generic executor (the Fig. 5 ablation).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../mbconv_types.h"
#include "ir.h"

namespace souffle {

struct MbPlan {
  bool on = false;
  std::string why_not;
  int x = -1, We = -1, se = -1, be = -1, sd = -1, bd = -1, W1 = -1, b1 = -1, W2 = -1, b2 = -1, Wp = -1, sp = -1,
      bp = -1, y = -1;
  int w[MB_MAX_TAPS], m[MB_MAX_TAPS];
  int H = 0, cin = 0, E = 0, k = 0, stride = 1, S = 0, cout = 0, residual = 0, grid = 0, num_sp = 0;
  int reuse = 0, pix_blk = 0;
  int64_t o_ctrl = 0, o_a = 0, o_d = 0, o_part = 0, o_pooled = 0, o_h = 0, o_acc = 0, total = 0;
};

void mbconv_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, MbPlan& mp);
std::string mbconv_describe(const MbPlan& mp);

}  // namespace souffle
