// Plain-data structures shared by the ResNeXt Bottleneck pattern planner (csrc/host/resnext.cpp) and its
// persistent kernel (csrc/kernels/resnext.cu).
//
// PAPER.md Table 2 (L1303): ResNeXt-101, 64 groups x 4d bottleneck width.  The block's TE program
// (models.resnext / oracle.graphs.resnext, pinned to torchvision's Bottleneck):
//   a = ReLU(BN(x W1^T))                                  1x1 convolution
//   c = sum_t [m_t * roll(a, -o_t)] grouped (x) W2_t      grouped 3x3 convolution: per tap one batched
//                                                         matmul over the G groups (cg channels each)
//   d = ReLU(BN(c[::s, ::s]))
//   y = ReLU(BN(d W3^T) + shortcut)                       shortcut x, or BN(x[::s, ::s] Wd^T)
// compiled to ONE persistent launch with two grid synchronisations (the 3x3 halo needs neighbouring
// pixels of a; the 1x1 convolution after it needs every channel of d).
#pragma once
#include <stdint.h>

namespace souffle {

enum { RX_THREADS = 256, RX_TAPS = 9, RX_MAX_TILES = 1024 };

struct RxParams {
  const float* x;                 // [H*H][cin]
  const float* W1;                // [w][cin]
  const float* s1;                // [w] BN scale / bias
  const float* b1;
  const float* W2[RX_TAPS];       // tap t = 3 i + j: [G][cg][cg] (out, in within the group)
  const float* m[RX_TAPS];        // tap t: [H*H] border mask (null for the centre tap)
  const float* s2;                // [w]
  const float* b2;
  const float* W3;                // [cout][w]
  const float* s3;                // [cout]
  const float* b3;
  const float* Wd;                // [cout][cin] projection shortcut (null: identity)
  const float* sd;                // [cout]
  const float* bd;
  float* y;                       // [Ho*Ho][cout] (also holds the projection shortcut between phases)
  float* a;                       // workspace [H*H][w]
  float* d;                       // workspace [Ho*Ho][w]
  unsigned* ctrl;                 // [0..1] grid barriers, [4] exit counter
  float* acc1;                    // split-K fp32 accumulators (zero between launches) of the 1x1 GEMM,
  float* acc2;                    // the projection and the second 1x1 GEMM
  float* acc3;
  unsigned* cnt;                  // [3][RX_MAX_TILES] per-tile split arrival counters (zero between launches)
  unsigned long long* prof;       // debug (SOUFFLE_RX_PROF): %globaltimer of CTA 0 at the phase boundaries [4]
  int32_t H, cin, w, G, stride, cout, pad0, pad1;
};

}  // namespace souffle
