// Plain-data structures shared by the host planner (csrc/host/mmoe.cpp) and the fused MMoE kernel
// (csrc/kernels/mmoe.cu).  PAPER.md Table 2 L1308 (MMoE), §6.1 horizontal transformation (the 8
// expert GEMMs and the 2 gate GEMMs share x and run as one fused GEMM), Table 5 (one kernel).
#pragma once
#include <stdint.h>
#include <vector_types.h>

namespace souffle {

// MMOE_CL: CTAs of the cluster variant (mmoe_cluster_kernel)
enum { MMOE_CL = 8, MMOE_SEG = 40, MMOE_THREADS = 1024, MMOE_MAX_E = 16, MMOE_MAX_T = 8, MMOE_MAX_B = 8, MMOE_MAX_SMEM = 200 * 1024 };

struct MmoeParams {
  const float* x;                  // [B][D]
  const void* We[MMOE_MAX_E];      // expert weights [De][D]
  const float* be[MMOE_MAX_E];     // [De]
  const void* Wg[MMOE_MAX_T];      // gate weights [E][D]
  const float* bg[MMOE_MAX_T];     // [E]
  const void* Wt[MMOE_MAX_T];      // tower hidden [Th][De]
  const float* bt[MMOE_MAX_T];     // [Th]
  const void* Wo[MMOE_MAX_T];      // tower output [1][Th]
  const float* bo[MMOE_MAX_T];     // [1]
  float* y[MMOE_MAX_T];            // outputs [B][1]
  int32_t B, D, E, De, T, Th;
  int32_t w_f32, pad;
  // parameter staging table, built on the host at workspace initialisation (pointers are known then;
  // a re-bind marks the plan dirty): seg[t * MMOE_SEG + j] = {src lo, src hi, smem byte offset, prefix
  // of 16-byte (t = 0, weights) or 4-byte (t = 1, vectors) units}, entry nseg[t] holds the total
  const uint4* seg;
  int32_t nseg[2];
};

}  // namespace souffle
