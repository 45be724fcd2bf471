// Pattern lowering for BERT encoder stacks (Table 2).
// When the whole TE program is a stack of post-LN BERT encoder layers with bf16 GEMM operands, the
// subprogram is executed by the specialised persistent kernel in kernels/bert.cu instead of the
// generic stage interpreter.  The match is strict: every TE of the program must belong to the
// pattern, with the exact semantics the kernel implements (scale 1/sqrt(d), max-subtracted softmax,
// erf GELU, biased-variance LayerNorm with the graph's eps); anything else falls back to the
// generic executor.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "ir.h"

namespace souffle {

struct BertLayerIds {
  int Wq = -1, bq = -1, Wk = -1, bk = -1, Wv = -1, bv = -1, Wo = -1, bo = -1, g1 = -1, be1 = -1;
  int W1 = -1, c1 = -1, W2 = -1, c2 = -1, g2 = -1, be2 = -1;
  int out = -1;        // the layer's output TE (LN2 result)
};

struct BertGemmCfg {
  int nt = 0, nsplit = 0, kchunks = 0, tiles_n = 0;
};

struct BertPlan {
  bool on = false;
  std::string why_not;           // reason the pattern was not used (describe())
  int X = -1, Y = -1;
  int S = 0, H = 0, heads = 0, d = 0, F = 0;
  double eps = 0.0;
  std::vector<BertLayerIds> layers;
  BertGemmCfg qkv, out, ffn1, ffn2;
  int num_sms = 0;
  bool pairs = false;             // QKV / FFN1 as cluster-pair split-K (kernels/bert.cu pair_tail)
  int nstages = 0;
  int nflags = 0;                 // point-to-point flags in the control block (kernels/bert.cu)
  // workspace layout (byte offsets from the workspace base)
  int64_t o_ctrl = 0, o_stages = 0, o_tmaps = 0, o_prof = 0;
  int64_t o_xb = 0, o_ctx = 0, o_l1b = 0, o_l1f = 0, o_xf = 0;
  int64_t o_h = 0, o_qk = 0, o_vt = 0, o_part_o = 0, o_part_2 = 0;
  int64_t o_consts = 0;          // packed per-layer fp32 vectors (bias / gamma / beta), refreshed by stage 0
  int64_t o_copies = 0;          // BCopy table: bound vector -> packed copy
  int64_t total = 0;
  int ncopies = 0, copy_total = 0;   // constant-refresh table (set at workspace init)
};

// Fills bp (bp.on = true) if g is a BERT encoder stack that the specialised kernel implements.
// The match is driven by the partition (§5.4 / §6.1): the kernel runs ONE subprogram, so the
// analysis must have put every TE into subprogram 0, and the [Q | K | V] horizontal GEMM is taken from
// the analysis' horizontal group of the three matmuls (N-concat, shared A operand).
void bert_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, BertPlan& bp);
std::string bert_describe(const BertPlan& bp);

}  // namespace souffle
