// Plain-data structures shared by the MBConv pattern planner (csrc/host/mbconv.cpp) and its persistent
// kernel (csrc/kernels/mbconv.cu).
//
// PAPER.md Fig. 5 / 6 (L1511-1564): "the sub-module is the building block of EfficientNet" -- the MBConv
// block, written as a TE program (models.mbconv / oracle.graphs.mbconv, pinned to torchvision):
//   a = SiLU(BN(x We^T))                                    1x1 expand convolution (if expand != 1)
//   d = SiLU(BN(sum_t m_t * roll(a, -o_t) * w_t))[::s, ::s] depthwise k x k convolution (rolled,
//                                                           border-masked taps), stride s
//   d = d * sigmoid(fc2(SiLU(fc1(mean(d)))))                squeeze-and-excitation
//   y = BN(d Wp^T) (+ x)                                    1x1 project convolution (+ residual)
// compiled to ONE persistent launch with four grid synchronisations (the one-relies-on-many
// dependencies: the depthwise halo, the pool, fc1, fc2).
#pragma once
#include <stdint.h>

namespace souffle {

enum { MB_THREADS = 256, MB_MAX_KS = 5, MB_MAX_TAPS = MB_MAX_KS * MB_MAX_KS, MB_MAX_E = 2048,
       MB_MAX_REUSE_SMEM = 160 * 1024 };

struct MbParams {
  const float* x;                 // [H*H][cin]
  const float* We;                // [E][cin]   (null: expand ratio 1, a = x)
  const float* se;                // [E] expand BN scale
  const float* be;                // [E] expand BN bias
  const float* w[MB_MAX_TAPS];    // tap t = i * k + j: [E] depthwise weights
  const float* m[MB_MAX_TAPS];    // tap t: [H*H] border mask (null for the centre tap)
  const float* sd;                // [E] depthwise BN scale
  const float* bd;                // [E]
  const float* W1;                // [S][E]
  const float* b1;                // [S]
  const float* W2;                // [E][S]
  const float* b2;                // [E]
  const float* Wp;                // [cout][E]
  const float* sp;                // [cout] project BN scale
  const float* bp;                // [cout]
  float* y;                       // [Ho*Ho][cout]
  float* a;                       // workspace [H*H][E] (expand output)
  float* d;                       // workspace [Ho*Ho][E] (depthwise output)
  float* pooled;                  // [E] channel sums of d (zero between launches)
  float* h;                       // [S]
  float* acc;                     // [Ho*Ho][cout] split-K accumulator of the project GEMM
  unsigned* ctrl;                 // [0..3] grid barriers, [5] exit counter
  unsigned long long* prof;       // debug (SOUFFLE_MB_PROF): %globaltimer of CTA 0 at the phase boundaries [8]
  int32_t H, cin, E, k, stride, S, cout, residual;
  int32_t reuse;     // 1: Fig. 5(d) data reuse (d block + Wp in shared memory), 0: d through L2
  int32_t pix_blk;   // reuse: output pixels per CTA
};

}  // namespace souffle
