// EfficientNet MBConv block (M0-M9) as ONE persistent kernel on sm_100a (Fig. 5(c), Fig. 6,
// L1511-1564; the TE program of csrc/mbconv_types.h, fp32 like the oracle):
//
//   1  expand      a = SiLU(x We^T * se + be)             32 x 32 output tiles over the grid  | sync
//   2  depthwise   d = SiLU(sum_t m_t[p] a[p + o_t] w_t * sd + bd) at the strided output pixels;
//                  the TE's roll is a cyclic shift, so the tap reads a at ((h + i - pad) mod H,
//                  (w + j - pad) mod H) and the border mask (an input) zeroes what wrapped around;
//                  per-CTA pool partial sums in a fixed order                          | sync
//   3  SE          pooled = sum of the partials / pixels | sync | h = SiLU(W1 pooled + b1) | sync |
//                  every CTA: g = sigmoid(W2 h + b2) for all channels (shared memory)
//   4  project     y = (d * g) Wp^T * sp + bp (+ x)       32 x 32 output tiles; the SE rescale is
//                  applied while the A tile is staged
//
// Four grid synchronisations -- the one-relies-on-many dependencies of the block (the depthwise halo
// needs neighbouring pixels of a, the pool needs every pixel, fc1 every channel, fc2 all of h) --
// plus one when the project GEMM splits K, and no other launch: the global-sync version of Fig. 5(c).  d goes through L2 (a d tile of all
// channels does not fit shared memory for the wide modules).
#include <cuda_runtime.h>
#include <stdint.h>

#include "../mbconv_types.h"
#include "ptx.cuh"

namespace souffle {
namespace mb {

__device__ __forceinline__ void grid_sync(const MbParams& P, int k) {
  __syncthreads();
  if (threadIdx.x == 0) {
    ptx::red_release_add(&P.ctrl[k], 1u);
    while (ptx::ld_acquire(&P.ctrl[k]) < gridDim.x) {
    }
  }
  __syncthreads();
}

__device__ __forceinline__ float sigm(float x) { return 1.f / (1.f + __expf(-x)); }
__device__ __forceinline__ float silu(float x) { return x * sigm(x); }

// C[m0.., n0..] (32 x 32) = sum_k A(m, k) B[n][k] over K; A(m, k) = Arow[m * lda + k] * (ascale ?
// ascale[k] : 1); epi(m, n, v) for the in-range outputs.  256 threads, 2 x 2 outputs each.
template <class Epi>
__device__ __forceinline__ void tile32(const float* A, int lda, const float* ascale, const float* B, int ldb, int M, int N,
                                       int kbeg, int kend, int m0, int n0, float (*As)[33], float (*Bs)[33], Epi epi) {
  const int tid = threadIdx.x, ty = tid >> 4, tx = tid & 15;
  float c00 = 0.f, c01 = 0.f, c10 = 0.f, c11 = 0.f;
  for (int k0 = kbeg; k0 < kend; k0 += 32) {
    __syncthreads();
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int e = tid + q * MB_THREADS, r = e >> 5, kk = e & 31, k = k0 + kk;
      float av = 0.f, bv = 0.f;
      if (m0 + r < M && k < kend) {
        av = __ldcg(A + (int64_t)(m0 + r) * lda + k);
        if (ascale) av *= ascale[k];
      }
      if (n0 + r < N && k < kend) bv = __ldg(B + (int64_t)(n0 + r) * ldb + k);
      As[r][kk] = av;
      Bs[r][kk] = bv;
    }
    __syncthreads();
#pragma unroll 8
    for (int kk = 0; kk < 32; ++kk) {
      const float a0 = As[ty * 2][kk], a1 = As[ty * 2 + 1][kk];
      const float b0 = Bs[tx * 2][kk], b1 = Bs[tx * 2 + 1][kk];
      c00 = fmaf(a0, b0, c00);
      c01 = fmaf(a0, b1, c01);
      c10 = fmaf(a1, b0, c10);
      c11 = fmaf(a1, b1, c11);
    }
  }
  const int m = m0 + ty * 2, n = n0 + tx * 2;
  if (m < M && n < N) epi(m, n, c00);
  if (m < M && n + 1 < N) epi(m, n + 1, c01);
  if (m + 1 < M && n < N) epi(m + 1, n, c10);
  if (m + 1 < M && n + 1 < N) epi(m + 1, n + 1, c11);
}

template <int KS>   // depthwise kernel size (0: any, loops not unrolled)
__global__ void __launch_bounds__(MB_THREADS, 1) mbconv_kernel(const __grid_constant__ MbParams P) {
  __shared__ float As[32][33], Bs[32][33];
  __shared__ float pool[MB_MAX_E];
  __shared__ float g[MB_MAX_E];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int H = P.H, E = P.E, k = P.k, s = P.stride, pad = k / 2;
  const int HW = H * H, Ho = H / s, HWo = Ho * Ho;
  const float* a = P.We ? P.a : P.x;   // expand ratio 1: the depthwise convolution reads x

  // ---- 1: expand convolution (+ BN + SiLU)
  if (P.We) {
    const int tm = (HW + 31) / 32, tn = (E + 31) / 32;
    for (int t = blockIdx.x; t < tm * tn; t += gridDim.x)
      tile32(P.x, P.cin, nullptr, P.We, P.cin, HW, E, 0, P.cin, (t / tn) * 32, (t % tn) * 32, As, Bs,
             [&](int m, int n, float v) { P.a[(int64_t)m * E + n] = silu(v * __ldg(P.se + n) + __ldg(P.be + n)); });
    grid_sync(P, 0);
  }
  // the project GEMM splits K over the idle CTAs when it has few output tiles (the narrow late modules:
  // 49 pixels x 1152 channels); its fp32 accumulator is cleared here, long before phase 4
  const int ptm = (HWo + 31) / 32, ptn = (P.cout + 31) / 32, ptiles = ptm * ptn;
  const int psplit = 2 * ptiles <= (int)gridDim.x ? min((int)gridDim.x / ptiles, (E + 31) / 32) : 1;
  if (psplit > 1)
    for (int i = blockIdx.x * MB_THREADS + tid; i < HWo * P.cout; i += gridDim.x * MB_THREADS) P.acc[i] = 0.f;
  // ---- 2: depthwise convolution (+ BN + SiLU) of this CTA's block of output pixels; (pixel, channel)
  // pairs are spread over all threads (consecutive threads: consecutive channels, coalesced), the taps
  // unrolled for the kernel sizes of the network (all loads of a pixel in flight together); pool
  // partial sums per CTA in shared memory
  {
    const int per = (HWo + gridDim.x - 1) / gridDim.x;
    const int q0 = blockIdx.x * per, q1 = min(HWo, q0 + per);
    for (int e = tid; e < E; e += MB_THREADS) pool[e] = 0.f;
    __syncthreads();
    for (int idx = tid; idx < (q1 - q0) * E; idx += MB_THREADS) {
      const int q = q0 + idx / E, e = idx % E;
      const int hs = (q / Ho) * s, ws = (q % Ho) * s;   // the pixel in the stride-1 grid
      const int kk = KS ? KS : k;
      float acc = 0.f;
#pragma unroll
      for (int i = 0; i < (KS ? KS : MB_MAX_KS); ++i) {
        if (!KS && i >= kk) break;
        const int hh = (hs + i - pad + H) % H;
#pragma unroll
        for (int j = 0; j < (KS ? KS : MB_MAX_KS); ++j) {
          if (!KS && j >= kk) break;
          const int t = i * kk + j, ww = (ws + j - pad + H) % H;
          float v = __ldcg(a + (int64_t)(hh * H + ww) * E + e);
          if (P.m[t]) v *= __ldg(P.m[t] + hs * H + ws);
          acc = fmaf(v, __ldg(P.w[t] + e), acc);
        }
      }
      const float dv = silu(acc * __ldg(P.sd + e) + __ldg(P.bd + e));
      P.d[(int64_t)q * E + e] = dv;
      atomicAdd(&pool[e], dv);
    }
    __syncthreads();
    for (int e = tid; e < E; e += MB_THREADS) P.part[(int64_t)blockIdx.x * E + e] = pool[e];
  }
  grid_sync(P, 1);
  // ---- 3: squeeze-and-excitation
  for (int e = blockIdx.x * MB_THREADS + tid; e < E; e += gridDim.x * MB_THREADS) {
    float sum = 0.f;
#pragma unroll 8
    for (int b = 0; b < (int)gridDim.x; ++b) sum += __ldcg(P.part + (int64_t)b * E + e);
    P.pooled[e] = sum / (float)HWo;
  }
  grid_sync(P, 2);
  for (int sq = blockIdx.x * (MB_THREADS / 32) + warp; sq < P.S; sq += gridDim.x * (MB_THREADS / 32)) {
    float acc = 0.f;
#pragma unroll 4
    for (int e = lane; e < E; e += 32) acc = fmaf(__ldg(P.W1 + (int64_t)sq * E + e), __ldcg(P.pooled + e), acc);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) P.h[sq] = silu(acc + __ldg(P.b1 + sq));
  }
  grid_sync(P, 3);
  for (int j = tid; j < P.S; j += MB_THREADS) pool[j] = __ldcg(P.h + j);   // h -> shared memory (pool is free)
  __syncthreads();
  for (int e = tid; e < E; e += MB_THREADS) {
    float acc = 0.f;
#pragma unroll 8
    for (int j = 0; j < P.S; ++j) acc = fmaf(__ldg(P.W2 + (int64_t)e * P.S + j), pool[j], acc);
    g[e] = sigm(acc + __ldg(P.b2 + e));
  }
  __syncthreads();
  // ---- 4: project convolution on the rescaled d (+ BN, + residual)
  auto finish = [&](int m, int n, float v) {
    float y = v * __ldg(P.sp + n) + __ldg(P.bp + n);
    if (P.residual) y += __ldg(P.x + (int64_t)m * P.cout + n);
    P.y[(int64_t)m * P.cout + n] = y;
  };
  if (psplit == 1) {
    for (int t = blockIdx.x; t < ptiles; t += gridDim.x)
      tile32(P.d, E, g, P.Wp, E, HWo, P.cout, 0, E, (t / ptn) * 32, (t % ptn) * 32, As, Bs, finish);
  } else {
    const int kper = ((E + psplit - 1) / psplit + 31) / 32 * 32;
    for (int w = blockIdx.x; w < ptiles * psplit; w += gridDim.x) {
      const int t = w / psplit, kb = (w % psplit) * kper;
      if (kb < E)
        tile32(P.d, E, g, P.Wp, E, HWo, P.cout, kb, min(E, kb + kper), (t / ptn) * 32, (t % ptn) * 32, As, Bs,
               [&](int m, int n, float v) { atomicAdd(P.acc + (int64_t)m * P.cout + n, v); });
    }
    grid_sync(P, 4);
    for (int i = blockIdx.x * MB_THREADS + tid; i < HWo * P.cout; i += gridDim.x * MB_THREADS)
      finish(i / P.cout, i % P.cout, __ldcg(P.acc + i));
  }
  // ---- exit: the last CTA resets the barrier counters for the next launch
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    if (atomicAdd(&P.ctrl[5], 1u) == gridDim.x - 1) {
      P.ctrl[0] = P.ctrl[1] = P.ctrl[2] = P.ctrl[3] = P.ctrl[4] = P.ctrl[5] = 0u;
      __threadfence();
    }
  }
}

}  // namespace mb

cudaError_t mbconv_launch(const MbParams& prm, int grid, cudaStream_t s) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(MB_THREADS);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;   // the grid barriers need every CTA co-resident
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  void (*fn)(MbParams) = prm.k == 3 ? mb::mbconv_kernel<3> : prm.k == 5 ? mb::mbconv_kernel<5> : mb::mbconv_kernel<0>;
  return cudaLaunchKernelEx(&cfg, fn, prm);
}

}  // namespace souffle
