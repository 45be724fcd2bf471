// Pattern lowering for Swin Transformers (Table 2; torchvision swin_b semantics, the
// TE program of models.swin).  When the whole TE program is a Swin Transformer with bf16 GEMM
// operands, window 7 and head dim 32, its fused subprograms run on the kernels of
// kernels/swin.cu instead of the generic stage interpreter.  The match is strict (every TE of the
// program, in the builder's order, with the exact semantics the kernels implement); anything else
// falls back to the generic executor.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../swin_types.h"
#include "ir.h"

namespace souffle {

struct SwinBlockIds {
  int g1 = -1, be1 = -1, Wqkv = -1, bqkv = -1, bias = -1, mask = -1, Wp = -1, bp = -1;
  int g2 = -1, be2 = -1, W1 = -1, b1 = -1, W2 = -1, b2 = -1;
  int stage = 0, shift = 0;
};
struct SwinMergeIds {
  int g = -1, be = -1, W = -1;
};

// one kernel launch of the plan (tensor maps are encoded at souffle_workspace_init)
struct SwinOp {
  int kind = 0;                 // SwOpKind
  SwGemm gemm{};
  SwAttn attn{};
  SwRow row{};
  SwIm2col im2col{};
  SwHead head{};
  SwBias bias{};
  int grid = 0;
  bool two_sm = false;          // GEMM on CTA pairs (sw_gemm2_kernel, cta_group::2)
  // tensor map requests: (buffer id, rows, cols, box rows, box cols, swizzle bytes); buffer ids are
  // workspace offsets (>= 0) or -(node + 1) for a bound tensor
  struct Map { int64_t buf; int64_t rows, cols; int box_rows, box_cols, swz; };
  Map maps[3];
  int nmaps = 0;
};

struct SwinPlan {
  bool on = false;
  std::string why_not;
  int B = 0, img = 0, patch = 0, C0 = 0, window = 0, classes = 0, mlp = 4;
  double eps = 0.0;
  std::vector<int> depths, heads;
  int X = -1, Y = -1, Wpe = -1, bpe = -1, gpe = -1, bepe = -1, gn = -1, ben = -1, Wh = -1, bh = -1;
  std::vector<SwinBlockIds> blocks;
  std::vector<SwinMergeIds> merges;
  // workspace layout (byte offsets)
  int64_t o_x0 = 0, o_x1 = 0, o_a = 0, o_ctx = 0, o_h = 0, o_q = 0, o_k = 0, o_vt = 0, o_pe = 0, o_wpad = 0;
  int64_t o_maps = 0, o_tab = 0, o_tabent = 0, tab_floats = 0, o_pool = 0, o_trace = 0, o_part = 0, o_cnt = 0, total = 0;
  std::vector<SwBiasEnt> tabent;   // score-bias table descriptors (pointers resolved at init)
  std::vector<int32_t> maps;    // host copy of the int32 index maps (uploaded at init)
  std::vector<SwinOp> ops;      // launch sequence (pointers resolved at init)
  int launches = 0;
  int num_sms = 148;
  void* graph_exec = nullptr;   // cudaGraphExec_t of the launch sequence (captured at init)
};

void swin_match(const Graph& g, const souffle_device_desc& dev, uint32_t flags, SwinPlan& sp);
std::string swin_describe(const SwinPlan& sp);

}  // namespace souffle
