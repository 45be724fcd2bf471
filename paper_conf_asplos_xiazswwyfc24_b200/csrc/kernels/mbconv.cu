// EfficientNet MBConv block (M0-M9) as ONE persistent kernel on sm_100a (Fig. 5(c), Fig. 6,
// L1511-1564; the TE program of csrc/mbconv_types.h, fp32 like the oracle):
//
//   1  expand      a = SiLU(x We^T * se + be)             64 x 64 (or 32 x 32) tiles over the grid | sync
//   2  depthwise   d = SiLU(sum_t m_t[p] a[p + o_t] w_t * sd + bd) at the strided output pixels;
//                  the TE's roll is a cyclic shift, so the tap reads a at ((h + i - pad) mod H,
//                  (w + j - pad) mod H) and the border mask (an input) zeroes what wrapped around;
//                  per-CTA pool partial sums in a fixed order                          | sync
//   3  SE          per-CTA pool partials added atomically | sync | h = SiLU(W1 mean + b1) | sync |
//                  g = sigmoid(W2 h + b2) for the channels each phase-4 task reads (shared memory)
//   4  project     y = (d * g) Wp^T * sp + bp (+ x)       64 x 64 / 32 x 32 tiles (split K when few); the SE rescale is
//                  applied while the A tile is staged
//
// Three grid synchronisations -- the one-relies-on-many dependencies of the block (the depthwise halo
// needs neighbouring pixels of a, the pool every pixel, the gates all of h) --
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
__device__ __forceinline__ void stamp(const MbParams& P, int k) {
  if (P.prof && blockIdx.x == 0 && threadIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    P.prof[k] = t;
  }
}
__device__ __forceinline__ float silu(float x) { return x * sigm(x); }
// L1-cached load of data written earlier in this launch by other CTAs: safe after the grid barrier (its
// acquire invalidates L1, and the data is not written again); the depthwise taps re-read each element
// of a up to k*k times from neighbouring pixels
__device__ __forceinline__ float ld_ca(const float* p) {
  float v;
  asm volatile("ld.global.ca.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}

// C[m0.., n0..] (BM x BN) = sum_k A(m, k) B[n][k] over [kbeg, kend); A(m, k) = A[m * lda + k] * (ascale ?
// ascale[k] : 1); epi(m, n, v) for the in-range outputs.  256 threads, (BM/16) x (BN/16) outputs each;
// K in slabs of 16 staged k-major in shared memory (a column of the tile is contiguous).
template <int BM, int BN, class Epi>
__device__ __forceinline__ void tile(const float* A, int lda, const float* ascale, const float* B, int ldb, int M, int N,
                                     int kbeg, int kend, int m0, int n0, float* sm, Epi epi) {
  constexpr int RM = BM / 16, RN = BN / 16;
  float(*As)[BM + 1] = reinterpret_cast<float(*)[BM + 1]>(sm);
  float(*Bs)[BN + 1] = reinterpret_cast<float(*)[BN + 1]>(sm + 16 * (BM + 1));
  const int tid = threadIdx.x, ty = tid >> 4, tx = tid & 15;
  float c[RM][RN];
#pragma unroll
  for (int i = 0; i < RM; ++i)
#pragma unroll
    for (int j = 0; j < RN; ++j) c[i][j] = 0.f;
  for (int k0 = kbeg; k0 < kend; k0 += 16) {
    __syncthreads();
#pragma unroll
    for (int q = 0; q < (BM * 16) / MB_THREADS; ++q) {
      const int e = tid + q * MB_THREADS, kk = e & 15, r = e >> 4, k = k0 + kk;
      float av = 0.f;
      if (m0 + r < M && k < kend) {
        av = __ldcg(A + (int64_t)(m0 + r) * lda + k);
        if (ascale) av *= ascale[k];
      }
      As[kk][r] = av;
    }
#pragma unroll
    for (int q = 0; q < (BN * 16) / MB_THREADS; ++q) {
      const int e = tid + q * MB_THREADS, kk = e & 15, r = e >> 4, k = k0 + kk;
      Bs[kk][r] = (n0 + r < N && k < kend) ? __ldg(B + (int64_t)(n0 + r) * ldb + k) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      float av[RM], bv[RN];
#pragma unroll
      for (int i = 0; i < RM; ++i) av[i] = As[kk][ty * RM + i];
#pragma unroll
      for (int j = 0; j < RN; ++j) bv[j] = Bs[kk][tx * RN + j];
#pragma unroll
      for (int i = 0; i < RM; ++i)
#pragma unroll
        for (int j = 0; j < RN; ++j) c[i][j] = fmaf(av[i], bv[j], c[i][j]);
    }
  }
#pragma unroll
  for (int i = 0; i < RM; ++i)
#pragma unroll
    for (int j = 0; j < RN; ++j) {
      const int m = m0 + ty * RM + i, n = n0 + tx * RN + j;
      if (m < M && n < N) epi(m, n, c[i][j]);
    }
}

// 64 x 64 tile with 4 x 4 outputs per thread: one float4 of A and of B per thread and 16-deep slab,
// the next slab's pair fetched into registers while the current one is multiplied, transposed into
// 16-byte-aligned k-major rows (68 floats) and read back as two 128-bit shared loads per 16 FMA.  A
// through L1 (written before the last grid barrier, never again in the launch), scaled by ascale[k]
// when given.  Needs lda and K multiples of 4 (every MBConv channel count is).
template <class Epi>
__device__ __forceinline__ void tile64(const float* A, int lda, const float* ascale, const float* B, int ldb, int M,
                                       int N, int kbeg, int kend, int m0, int n0, float* sm, Epi epi) {
  constexpr int LD = 68;
  float(*As)[LD] = reinterpret_cast<float(*)[LD]>(sm);
  float(*Bs)[LD] = reinterpret_cast<float(*)[LD]>(sm + 16 * LD);
  const int tid = threadIdx.x, ty = tid >> 4, tx = tid & 15;
  const int lr = tid & 63, lq = tid >> 6;
  const bool aok = m0 + lr < M, bok = n0 + lr < N;
  const float* ap = A + (int64_t)(aok ? m0 + lr : 0) * lda + 4 * lq;
  const float* bp = B + (int64_t)(bok ? n0 + lr : 0) * ldb + 4 * lq;
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
  auto lda4 = [&](int k0) {
    if (!aok || k0 + 4 * lq >= kend) return z4;
    float4 v;
    asm volatile("ld.global.ca.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(ap + k0));
    if (ascale) {
      const int k = k0 + 4 * lq;
      v.x *= ascale[k]; v.y *= ascale[k + 1]; v.z *= ascale[k + 2]; v.w *= ascale[k + 3];
    }
    return v;
  };
  auto ldb4 = [&](int k0) { return (!bok || k0 + 4 * lq >= kend) ? z4 : __ldg(reinterpret_cast<const float4*>(bp + k0)); };
  float c[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) c[i][j] = 0.f;
  float4 an = lda4(kbeg), bn = ldb4(kbeg);
  for (int k0 = kbeg; k0 < kend; k0 += 16) {
    __syncthreads();
    As[4 * lq + 0][lr] = an.x; As[4 * lq + 1][lr] = an.y; As[4 * lq + 2][lr] = an.z; As[4 * lq + 3][lr] = an.w;
    Bs[4 * lq + 0][lr] = bn.x; Bs[4 * lq + 1][lr] = bn.y; Bs[4 * lq + 2][lr] = bn.z; Bs[4 * lq + 3][lr] = bn.w;
    __syncthreads();
    if (k0 + 16 < kend) {
      an = lda4(k0 + 16);
      bn = ldb4(k0 + 16);
    }
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      const float4 a4 = *reinterpret_cast<const float4*>(&As[kk][4 * ty]);
      const float4 b4 = *reinterpret_cast<const float4*>(&Bs[kk][4 * tx]);
      const float av[4] = {a4.x, a4.y, a4.z, a4.w}, bv[4] = {b4.x, b4.y, b4.z, b4.w};
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) c[i][j] = fmaf(av[i], bv[j], c[i][j]);
    }
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int m = m0 + 4 * ty + i, n = n0 + 4 * tx + j;
      if (m < M && n < N) epi(m, n, c[i][j]);
    }
}

// a GEMM phase over output tiles: 64 x 64 tiles when they fill half the grid, else 32 x 32
template <class Epi>
__device__ __forceinline__ void gemm_phase(const float* A, int lda, const float* ascale, const float* B, int M, int N, int K,
                                           float* sm, Epi epi) {
  const int t64 = ((M + 63) / 64) * ((N + 63) / 64);
  if (2 * t64 >= (int)gridDim.x) {
    const int tn = (N + 63) / 64;
    for (int t = blockIdx.x; t < t64; t += gridDim.x)
      tile64(A, lda, ascale, B, K, M, N, 0, K, (t / tn) * 64, (t % tn) * 64, sm, epi);
  } else {
    const int tn = (N + 31) / 32, t32 = ((M + 31) / 32) * tn;
    for (int t = blockIdx.x; t < t32; t += gridDim.x)
      tile<32, 32>(A, lda, ascale, B, K, M, N, 0, K, (t / tn) * 32, (t % tn) * 32, sm, epi);
  }
}

template <int KS>   // depthwise kernel size (0: any, loops not unrolled)
__global__ void __launch_bounds__(MB_THREADS, 1) mbconv_kernel(const __grid_constant__ MbParams P) {
  __shared__ __align__(16) float tsm[2 * 16 * 68];   // GEMM operand slabs
  __shared__ float pool[MB_MAX_E];
  __shared__ float g[MB_MAX_E];
  extern __shared__ float dyn[];       // data reuse: [pix_blk][E] depthwise output, then [cout][E + 1] Wp
  float* d_s = dyn;
  float* wp_s = dyn + P.pix_blk * P.E;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int H = P.H, E = P.E, k = P.k, s = P.stride, pad = k / 2;
  const int HW = H * H, Ho = H / s, HWo = Ho * Ho;
  const float* a = P.We ? P.a : P.x;   // expand ratio 1: the depthwise convolution reads x

  stamp(P, 0);
  // ---- 1: expand convolution (+ BN + SiLU)
  if (P.We) {
    gemm_phase(P.x, P.cin, nullptr, P.We, HW, E, P.cin, tsm,
               [&](int m, int n, float v) { P.a[(int64_t)m * E + n] = silu(v * __ldg(P.se + n) + __ldg(P.be + n)); });
    stamp(P, 1);
    grid_sync(P, 0);
  }
  stamp(P, 2);
  // the project GEMM splits K over the idle CTAs when it has few output tiles (the narrow late modules:
  // 49 pixels x 1152 channels); its fp32 accumulator is cleared here, long before phase 4
  const int ptm = (HWo + 31) / 32, ptn = (P.cout + 31) / 32, ptiles = ptm * ptn;
  const int psplit = !P.reuse && 2 * ptiles <= (int)gridDim.x ? min((int)gridDim.x / ptiles, (E + 31) / 32) : 1;
  if (psplit > 1)
    for (int i = blockIdx.x * MB_THREADS + tid; i < HWo * P.cout; i += gridDim.x * MB_THREADS) P.acc[i] = 0.f;
  // ---- 2: depthwise convolution (+ BN + SiLU) of this CTA's block of output pixels; (pixel, channel)
  // pairs are spread over all threads (consecutive threads: consecutive channels, coalesced), the taps
  // unrolled for the kernel sizes of the network (all loads of a pixel in flight together); pool
  // partial sums per CTA in shared memory
  {
    // the (pixel, channel) pairs of the whole output split evenly over the grid (a few wide pixels,
    // e.g. 7 x 7 x 1152, still keep every CTA busy)
    // (data reuse: whole pixel blocks, so that this CTA's d block stays in its shared memory)
    const int64_t total = (int64_t)HWo * E;
    const int64_t per = P.reuse ? (int64_t)P.pix_blk * E : (total + gridDim.x - 1) / gridDim.x;
    const int64_t i0 = blockIdx.x * per, i1 = min(total, i0 + per);
    for (int e = tid; e < E; e += MB_THREADS) pool[e] = 0.f;
    __syncthreads();
#pragma unroll 2
    for (int64_t idx = i0 + tid; idx < i1; idx += MB_THREADS) {
      const int q = (int)(idx / E), e = (int)(idx % E);
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
          float v = ld_ca(a + (int64_t)(hh * H + ww) * E + e);
          if (P.m[t]) v *= __ldg(P.m[t] + hs * H + ws);
          acc = fmaf(v, __ldg(P.w[t] + e), acc);
        }
      }
      const float dv = silu(acc * __ldg(P.sd + e) + __ldg(P.bd + e));
      if (P.reuse) d_s[idx - i0] = dv;
      else P.d[(int64_t)q * E + e] = dv;
      atomicAdd(&pool[e], dv);
    }
    __syncthreads();
    // this CTA's pool partials straight into the channel sums (fp32 atomics; pooled is zero at entry:
    // workspace initialisation, then the last CTA of every launch clears it)
    if (i0 < i1)
      for (int e = tid; e < E; e += MB_THREADS) atomicAdd(P.pooled + e, pool[e]);
  }
  stamp(P, 3);
  grid_sync(P, 1);
  stamp(P, 4);
  // ---- 3: squeeze-and-excitation: h = SiLU(W1 mean + b1) (warp per squeeze channel)
  for (int sq = blockIdx.x * (MB_THREADS / 32) + warp; sq < P.S; sq += gridDim.x * (MB_THREADS / 32)) {
    float acc = 0.f;
#pragma unroll 4
    for (int e = lane; e < E; e += 32) acc = fmaf(__ldg(P.W1 + (int64_t)sq * E + e), __ldcg(P.pooled + e), acc);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) P.h[sq] = silu(acc / (float)HWo + __ldg(P.b1 + sq));
  }
  grid_sync(P, 2);
  stamp(P, 5);
  for (int j = tid; j < P.S; j += MB_THREADS) pool[j] = __ldcg(P.h + j);   // h -> shared memory (pool is free)
  __syncthreads();
  // excitation gates g[e] = sigmoid(W2[e] . h + b2[e]) for the channels [e0, e1) a phase-4 task reads
  auto gates = [&](int e0, int e1) {
    __syncthreads();
    for (int e = e0 + tid; e < e1; e += MB_THREADS) {
      float acc = 0.f;
#pragma unroll 8
      for (int j = 0; j < P.S; ++j) acc = fmaf(__ldg(P.W2 + (int64_t)e * P.S + j), pool[j], acc);
      g[e] = sigm(acc + __ldg(P.b2 + e));
    }
    __syncthreads();
  };
  // ---- 4: project convolution on the rescaled d (+ BN, + residual)
  if (P.reuse) {
    // ---- 4 (data reuse, Fig. 5(d)): this CTA's own pixels, d from shared memory, Wp staged beside it
    const int q0 = blockIdx.x * P.pix_blk, nq = min(P.pix_blk, HWo - q0);
    if (nq > 0) {
      gates(0, E);
      for (int i = tid; i < P.cout * E; i += MB_THREADS) wp_s[(i / E) * (E + 1) + i % E] = __ldg(P.Wp + i);
      for (int i = tid; i < nq * E; i += MB_THREADS) d_s[i] *= g[i % E];
      __syncthreads();
      for (int o = tid; o < nq * P.cout; o += MB_THREADS) {
        const int qq = o / P.cout, n = o % P.cout;
        const float* dr = d_s + qq * E;
        const float* wr = wp_s + n * (E + 1);   // padded rows: consecutive n on distinct banks
        float acc = 0.f;
#pragma unroll 4
        for (int e = 0; e < E; ++e) acc = fmaf(dr[e], wr[e], acc);
        const int m = q0 + qq;
        float y = acc * __ldg(P.sp + n) + __ldg(P.bp + n);
        if (P.residual) y += __ldg(P.x + (int64_t)m * P.cout + n);
        P.y[(int64_t)m * P.cout + n] = y;
      }
    }
  } else {
  auto finish = [&](int m, int n, float v) {
    float y = v * __ldg(P.sp + n) + __ldg(P.bp + n);
    if (P.residual) y += __ldg(P.x + (int64_t)m * P.cout + n);
    P.y[(int64_t)m * P.cout + n] = y;
  };
  if (psplit == 1) {
    if ((int)blockIdx.x < ptiles) gates(0, E);
    gemm_phase(P.d, E, g, P.Wp, HWo, P.cout, E, tsm, finish);
  } else {
    // split K: a task (tile, K slice) needs only its slice's gates (the late modules: the W2 rows of
    // 1152 channels are read once over the grid, not once per CTA)
    const int kper = ((E + psplit - 1) / psplit + 31) / 32 * 32;
    for (int w = blockIdx.x; w < ptiles * psplit; w += gridDim.x) {
      const int t = w / psplit, kb = (w % psplit) * kper;
      if (kb >= E) continue;
      gates(kb, min(E, kb + kper));
      tile<32, 32>(P.d, E, g, P.Wp, E, HWo, P.cout, kb, min(E, kb + kper), (t / ptn) * 32, (t % ptn) * 32, tsm,
                   [&](int m, int n, float v) { atomicAdd(P.acc + (int64_t)m * P.cout + n, v); });
    }
    grid_sync(P, 3);
    for (int i = blockIdx.x * MB_THREADS + tid; i < HWo * P.cout; i += gridDim.x * MB_THREADS)
      finish(i / P.cout, i % P.cout, __ldcg(P.acc + i));
  }
  }
  stamp(P, 6);
  // ---- exit: the last CTA resets the barrier counters and the pooled sums for the next launch
  __syncthreads();
  __shared__ int last;
  if (tid == 0) {
    __threadfence();
    last = atomicAdd(&P.ctrl[5], 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (last) {
    __threadfence();
    for (int e = tid; e < E; e += MB_THREADS) P.pooled[e] = 0.f;
    if (tid == 0) P.ctrl[0] = P.ctrl[1] = P.ctrl[2] = P.ctrl[3] = P.ctrl[4] = P.ctrl[5] = 0u;
    __threadfence();
  }
}

}  // namespace mb

size_t mbconv_reuse_smem(int pix_blk, int E, int cout) { return 4 * ((size_t)pix_blk * E + (size_t)cout * (E + 1)); }

cudaError_t mbconv_launch(const MbParams& prm, int grid, cudaStream_t s) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(MB_THREADS);
  cfg.dynamicSmemBytes = prm.reuse ? mbconv_reuse_smem(prm.pix_blk, prm.E, prm.cout) : 0;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;   // the grid barriers need every CTA co-resident
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  void (*fn)(MbParams) = prm.k == 3 ? mb::mbconv_kernel<3> : prm.k == 5 ? mb::mbconv_kernel<5> : mb::mbconv_kernel<0>;
  if (prm.reuse) {
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, MB_MAX_REUSE_SMEM);
    if (e != cudaSuccess) return e;
  }
  return cudaLaunchKernelEx(&cfg, fn, prm);
}

}  // namespace souffle
