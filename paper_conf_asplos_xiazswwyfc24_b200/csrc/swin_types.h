// Plain-data structures shared by the Swin pattern planner (csrc/host/swin.cpp) and its sm_100a
// kernels (csrc/kernels/swin.cu).
//
// When the partitioned TE program is a torchvision-semantics Swin Transformer (Table 2
// L1305; the TE program of models.swin), each fused subprogram of a block runs on a kernel written
// for its pattern (§6: horizontal + vertical transformations, reductions fused into their
// consumers):
//   ROW   LayerNorm of a token row gathered through the block's index maps (cyclic shift + window
//         partition, §6.2 quasi-affine maps; or the 2x2 patch-merge gather), bf16 GEMM operand out
//   GEMM  persistent tcgen05 GEMM (TMA ring, TMEM double-buffered accumulator, warp-specialised)
//         with the consumer chain in the epilogue: +bias, q-scale and the QKV reshape / permute /
//         slice maps folded into a scatter (QKV); +bias + residual through the window-reverse +
//         reverse-shift map (proj, FC2); +bias + erf-GELU (FC1); plain (patch merge / embed)
//   ATTN  window attention of two (window, head) units per M=128 tcgen05 tile: S = Q K^T (+ the
//         relative-position bias, + the shifted-window mask), fp32 softmax in registers, P V
//   HEAD  final LayerNorm + mean pool + classifier (one CTA per image)
#pragma once
#include <stdint.h>

namespace souffle {

enum SwOpKind : int32_t { SW_IM2COL = 0, SW_ROW = 1, SW_GEMM = 2, SW_ATTN = 3, SW_HEAD = 4, SW_BIAS = 5, SW_POOL = 6 };
enum SwEpi : int32_t { SWE_F32 = 0, SWE_GELU = 1, SWE_RESID = 2, SWE_QKV = 3 };

enum {
  SW_GEMM_THREADS = 320,      // warp 0 TMA producer, warp 1 MMA issuer, warps 2-9 epilogue (2 per
                              // TMEM lane quarter, interleaved 32-column chunks; 12 epilogue warps
                              // measured slower: register cap 128 -> spills)
  SW_ATTN_THREADS = 128,      // one thread per row of the M = 128 tile (two 64-row units)
  SW_ROW_THREADS = 256,       // 8 warps, one token row per warp
  SW_WIN_ROWS = 64,           // a (window, head) unit: 49 tokens padded to 64 rows
  SW_TAB = 2404,              // floats per (window, head) score-bias tile: 49 x 49 + 3 (16-byte multiple)
};

// one GEMM launch: C[M, N] = A[M, K] W[N, K]^T (bf16 operands, fp32 accumulate) + epilogue
struct SwGemm {
  int32_t M, N, K, BN;        // K % 64 == 0, N % BN == 0, BN in {64, 128, 256}
  int32_t epi, stages;        // SwEpi; TMA ring depth
  const float* bias;          // [N] or null
  float* out_f;               // SWE_F32: [M][N]; SWE_RESID: residual stream x [tokens][N] (+=)
  uint16_t* out_b;            // SWE_GELU: bf16 [M][N]
  const int32_t* rowmap;      // SWE_RESID: GEMM row (window order) -> token row; null = identity
  // SWE_QKV: columns [0, C) = q (scaled), [C, 2C) = k, [2C, 3C) = v of a [tokens, 3C] GEMM whose
  // rows are in window order (row = window * 49 + i).  q, k: [units][64][32] bf16, unit = window *
  // heads + head; vt: [units][32][64] bf16 (V transposed, keys contiguous)
  uint16_t *q, *k, *vt;
  int32_t C, heads, L2;       // L2 = window tokens (49)
  float qscale;
  // split-K (small M, e.g. batch 1: too few output tiles to occupy the SMs): unit = tile * splits +
  // split covers K chunks [split * nk / splits, ...); the fp32 partials go to part[unit][128][BN],
  // the `splits` CTAs of a tile meet on cnt[tile] and each reduces 128 / splits rows (fixed split
  // order: deterministic) through the fused epilogue; cnt[tiles + tile] counts the finished ones
  int32_t splits;             // 1 = no split
  float* part;
  unsigned* cnt;
  unsigned long long* trace;  // debug: %globaltimer at the start of launch `op` (CTA 0), or null
  int32_t op;
  int32_t direct;             // study: 1 = epilogue stores straight from registers (no staging tile)
};

// window attention over `units` (window, head) pairs, two per CTA iteration.  The additive score
// terms come from a per-block table tab[nW][heads][SW_TAB] = relative-position bias (+ shifted-window
// mask) built by sw_bias_kernel at the start of every run (nW = 1 for unshifted blocks), so a pair's
// two tiles are one contiguous bulk copy into shared memory
struct SwAttn {
  int32_t units, heads, nW, L2; // nW: windows per image in the table (window index = window % nW)
  const float* tab;
  uint16_t* ctx;                // bf16 [windows * L2][heads * 32] (window order)
  int32_t C;
  unsigned long long* trace;
  int32_t op;
};

// one block's score-bias table: dst[w][h][i * L2 + j] = bias[h][i][j] + (mask ? mask[w][i][j] : 0)
struct SwBiasEnt {
  const float* bias;
  const float* mask;
  float* dst;
  int32_t heads, nW, first, pad;   // first: element offset of this table in the concatenation
};
struct SwBias {
  const SwBiasEnt* ent;
  int32_t n, total, L2, op;
  unsigned long long* trace;
};

// LayerNorm of gathered rows: out[r] = LN(concat_s x[src[r * nsrc + s]]) * gamma + beta
struct SwRow {
  int32_t rows, cols, nsrc;     // cols = nsrc * C_in (<= 1024)
  const float* x;               // fp32 [tokens][C_in]
  const int32_t* src;           // [rows][nsrc] source token rows; null = identity (nsrc = 1)
  const float* gamma;
  const float* beta;
  float eps;
  uint16_t* out_b;              // bf16 [rows][cols] (GEMM A operand), or null
  float* out_f;                 // fp32 [rows][cols], or null
  unsigned long long* trace;
  int32_t op;
};

// patch-embedding im2col: image [B][3][H][W] fp32 -> bf16 [B * R * R][64] (48 used, cols =
// c * 16 + kh * 4 + kw, zero padded), plus the [C][48] weight padded to [C][64] bf16
struct SwIm2col {
  int32_t B, img, p, R, C;
  const float* image;
  uint16_t* out;
  const uint16_t* w;            // bound Wpe [C][48] (bf16)
  uint16_t* wpad;               // [C][64]
  unsigned long long* trace;
  int32_t op;
};

// final LayerNorm + mean over the L tokens of each image (sw_pool_kernel, one CTA per image; the
// mean is rounded to bf16: it is a matmul operand), then the classifier (sw_head_kernel, a warp per
// class over all images; bf16 operands, fp32 accumulate)
struct SwHead {
  int32_t B, L, C, classes;
  const float* x;               // fp32 [B * L][C]
  const float* gamma;
  const float* beta;
  float eps;
  const uint16_t* W;            // bf16 [classes][C]
  const float* bias;            // [classes]
  float* out;                   // fp32 [B][classes]
  float* pooled;                // fp32 [B][C] workspace (bf16-representable values)
  unsigned long long* trace;
  int32_t op;
};

}  // namespace souffle
