// Pattern lowering for multi-gate mixture-of-experts (Table 2): when the whole TE
// program is the MMoE built by models.mmoe (experts Linear+ReLU, per-task softmax gates, gated sum,
// towers Linear+ReLU -> Linear), it runs on the single-CTA fused kernel in kernels/mmoe.cu.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "ir.h"

namespace souffle {

struct MmoePlan {
  bool on = false;
  std::string why_not;
  int B = 0, D = 0, E = 0, De = 0, T = 0, Th = 0, w_f32 = 0;
  int x = -1;
  std::vector<int> We, be, Wg, bg, Wt, bt, Wo, bo, y;
  int nseg[2] = {0, 0};   // staging-table segments (set at workspace initialisation)
};

// driven by the partition: ONE subprogram (Table 5), and the expert and gate matmuls that read x form the
// analysis' N-concat horizontal group (§6.1) that the kernel's fused expert + gate GEMM implements
void mmoe_match(const Graph& g, const Analysis& an, uint32_t flags, MmoePlan& mp);
std::string mmoe_describe(const MmoePlan& mp);

}  // namespace souffle
