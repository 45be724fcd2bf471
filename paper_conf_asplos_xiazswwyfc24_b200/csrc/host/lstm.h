// Pattern lowering for stacked LSTMs (Table 2, §8.4): when the whole TE
// program is the unrolled torch.nn.LSTM recurrence built by models.lstm (gates i, f, g, o; b_ih and
// b_hh; fp32-precision GEMVs), it runs on the persistent wavefront kernel in kernels/lstm.cu.
// The match is strict (every TE accounted for, exact op order and operands); anything else falls
// back to the generic executor.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "ir.h"

namespace souffle {

struct LstmPlan {
  bool on = false;
  std::string why_not;
  int T = 0, L = 0, H = 0, I = 0, NP = 0, K_max = 0, w_f32 = 0;
  int reg = 0;   // 1: register-resident GEMV (lstm_reg_kernel), 0: weights in shared memory
  int X = -1;
  std::vector<int> W, U, bi, bh, h0, c0;   // per layer
  std::vector<int> top;                    // [T] output nodes (last layer h at t)
  std::vector<int> hn, cn;                 // [L] final-state output nodes
  // workspace layout
  int64_t o_gen = 0, o_layers = 0, o_top = 0, o_hbuf = 0, o_prof = 0, total = 0;
};

// driven by the partition: the analysis must have put every TE in ONE subprogram (Table 5: LSTM runs as
// one kernel) and found the reuse of every layer's W_ih / W_hh across the T steps (§5.1; W_hh temporal)
// that the kernel's on-chip weights implement
void lstm_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, LstmPlan& lp);
std::string lstm_describe(const LstmPlan& lp);

}  // namespace souffle
