// Plain-data structures shared by the host planner (csrc/host/lstm.cpp) and the persistent LSTM
// kernel (csrc/kernels/lstm.cu).
//
// PAPER.md §8.4: a stacked LSTM is one subprogram; Souffle keeps every cell's
// weights on chip across all time steps and synchronises the wavefront globally instead of
// relaunching (Table 6: 1911 MB of weight traffic for Rammer vs ~21 MB for Souffle).  Here layer l
// is owned by NP CTAs; CTA (l, p) keeps the 4*32 gate rows of hidden units [32p, 32p+32) of
// [W_ih | W_hh] in shared memory for the whole sequence and runs the cells (l, 0..T-1).  The
// wavefront dependencies (l, t-1) -> (l, t) and (l-1, t) -> (l, t) are carried by the data itself:
// every published h value is a 64-bit word (fp32 value, 32-bit tag = step of this run), so a
// consumer's single L2 round trip both detects readiness and fetches the operand (no fence, no
// separate flag; the "LL" low-latency protocol idea), and no grid barrier is involved.
#pragma once
#include <stdint.h>

namespace souffle {

enum { LSTM_THREADS = 512, LSTM_UNITS = 32, LSTM_ROWS = 4 * LSTM_UNITS, LSTM_MAX_SMEM = 200 * 1024 };
// register-resident GEMV variant (lstm_reg_kernel): warp w owns rows 5 (w % 4) .. + 4 of gate w / 4 over
// all K <= 512 columns (16 per lane), so a CTA holds <= 20 units and its weights in fp32 registers
enum { LSTM_REG_K = 512, LSTM_REG_RPW = 5, LSTM_REG_UNITS = 4 * LSTM_REG_RPW };

struct LstmLayer {
  const void* W;        // W_ih [4H][I_l] (bf16 or fp32, row-major)
  const void* U;        // W_hh [4H][H]
  const float* b_ih;    // [4H]
  const float* b_hh;    // [4H]
  const float* h0;      // [H]
  const float* c0;      // [H]
  float* h_n;           // [H] final hidden state (output)
  float* c_n;           // [H] final cell state (output)
  int32_t in_dim, pad;
};

struct LstmParams {
  const LstmLayer* layers;
  const float* X;        // [T][I_0]
  float* const* top;     // [T] output pointers: h of the last layer at step t ([H] each)
  uint2* hbuf;           // [L][T][H] (value bits, tag) of every hidden state, written exactly once per run
  unsigned int* gen;     // [0]: run generation (tags of this run are gen * (T + 1) + t + 1); [1]: exit counter
  int32_t L, T, H, NP;
  int32_t w_f32;         // 1: fp32 weights in smem, 0: bf16
  int32_t K_max;         // max_l (I_l + H): row length of the smem weight tile
  unsigned long long* prof;   // debug: per-step timestamps of CTA prof_cta ([T][4]), null if off
  int32_t prof_cta;
  int32_t reg;           // 1: weights resident in registers (lstm_reg_kernel), 0: in shared memory
};

}  // namespace souffle
