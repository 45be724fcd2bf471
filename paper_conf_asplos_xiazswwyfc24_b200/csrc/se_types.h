// Plain-data structures shared by the squeeze-and-excitation pattern planner (csrc/host/se.cpp) and
// its persistent kernel (csrc/kernels/se.cu).
//
// PAPER.md Fig. 5 / Fig. 6 (L1511-1564): the EfficientNet sub-module M0-M9 -- global average pool
// (one-relies-on-many), two GEMVs with SiLU / Sigmoid, and the channel-wise rescale of the same input
// -- compiled (c) to ONE kernel with global synchronisation and (d) with the input tensor reused from
// shared memory across the pool and the rescale ("data reuse", §6.5 tensor reuse L1205-1212).
#pragma once
#include <stdint.h>

namespace souffle {

enum { SE_THREADS = 256, SE_MAX_TILE_FLOATS = 40 * 1024 };   // x tile kept on chip: <= 160 KB

struct SeParams {
  const float* x;        // [HW][C]
  const float* W1;       // [S][C]
  const float* b1;       // [S]
  const float* W2;       // [C][S]
  const float* b2;       // [C]
  float* y;              // [HW][C]
  float* part;           // [nrb][C] per-row-block channel sums (workspace)
  float* pooled;         // [C]
  float* h;              // [S]
  unsigned* ctrl;        // [0..2] grid barriers, [3] exit counter
  int32_t HW, C, S;
  int32_t nrb, ncb, rows, cbw;   // row blocks, channel blocks, rows per row block, channels per block
  int32_t reuse;         // 1: the x tile stays in shared memory between the pool and the rescale
  int32_t pad;
};

}  // namespace souffle
