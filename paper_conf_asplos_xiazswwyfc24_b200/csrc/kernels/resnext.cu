// ResNeXt Bottleneck block (Table 2: ResNeXt-101, 64 groups x 4d) as ONE persistent kernel on
// sm_100a (the TE program of csrc/resnext_types.h, fp32 like the oracle):
//
//   1  a = ReLU(x W1^T * s1 + b1)                 64 x 64 (or 32 x 32) tiles over the grid, and the
//      projection shortcut y = x[::s, ::s] Wd^T * sd + bd (when the shape changes)        | sync
//   2  d = ReLU(sum_t m_t[p] sum_i W2_t[g][o][i] a[p + o_t][g cg + i] * s2 + b2) at the strided output
//      pixels: the grouped 3x3 convolution; the TE's roll is a cyclic shift, so tap t reads a at
//      ((h + i - 1) mod H, (w + j - 1) mod H) and the border mask (an input) zeroes what wrapped
//      around; one thread per (pixel, output channel), float4 loads along the group's channels | sync
//   3  y = ReLU(d W3^T * s3 + b3 + shortcut)       (shortcut: x, or the projection from phase 1)
//
// Two grid synchronisations -- the one-relies-on-many dependencies of the block (the 3x3 halo needs
// neighbouring pixels of a, the second 1x1 convolution every channel of d) -- and no other launch.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../resnext_types.h"
#include "ptx.cuh"

namespace souffle {
namespace rx {

__device__ __forceinline__ void grid_sync(const RxParams& P, int k) {
  __syncthreads();
  if (threadIdx.x == 0) {
    ptx::red_release_add(&P.ctrl[k], 1u);
    while (ptx::ld_acquire(&P.ctrl[k]) < gridDim.x) {
    }
  }
  __syncthreads();
}
__device__ __forceinline__ void stamp(const RxParams& P, int k) {
  if (P.prof && blockIdx.x == 0 && threadIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    P.prof[k] = t;
  }
}
// L1-cached load of data written earlier in this launch by other CTAs: safe after the grid barrier (its
// acquire invalidates L1, and the data is not written again); the 3x3 taps re-read a up to 9 times
__device__ __forceinline__ float4 ld_ca4(const float* p) {
  float4 v;
  asm volatile("ld.global.ca.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}

// C[m0.., n0..] (BM x BN) = sum_k A(arow(m), k) B[n][k]; epi(m, n, v) for the in-range outputs.  256
// threads, (BM/16) x (BN/16) outputs each; K in slabs of 16 staged k-major in shared memory.
template <int BM, int BN, class Row, class Epi>
__device__ __forceinline__ void tile(const float* A, int lda, Row arow, const float* B, int M, int N, int K, int kbeg,
                                     int kend, int m0, int n0, float* sm, Epi epi) {
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
    for (int q = 0; q < (BM * 16) / RX_THREADS; ++q) {
      const int e = tid + q * RX_THREADS, kk = e & 15, r = e >> 4, k = k0 + kk;
      As[kk][r] = (m0 + r < M && k < kend) ? __ldcg(A + (int64_t)arow(m0 + r) * lda + k) : 0.f;
    }
#pragma unroll
    for (int q = 0; q < (BN * 16) / RX_THREADS; ++q) {
      const int e = tid + q * RX_THREADS, kk = e & 15, r = e >> 4, k = k0 + kk;
      Bs[kk][r] = (n0 + r < N && k < kend) ? __ldg(B + (int64_t)(n0 + r) * K + k) : 0.f;
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

// 64 x 64 tile, 4 x 4 outputs per thread, K in slabs of 16: each thread loads one float4 of A and of B
// per slab (the next slab's pair is fetched into registers while the current one is multiplied) and
// stores it transposed (k-major rows of 68 floats: 16-byte aligned, conflict-free stores), and every
// k step reads its 4 A and 4 B values as two 128-bit shared loads (2 loads per 16 FMA).  Requires
// lda, K, kbeg, kend multiples of 4 (the matcher checks 16).  A through L1 (ld.global.ca: the input x,
// or d written before the last grid barrier, never written again in the launch).
template <class Row, class Epi>
__device__ __forceinline__ void tile64(const float* A, int lda, Row arow, const float* B, int M, int N, int K, int kbeg,
                                       int kend, int m0, int n0, float* sm, Epi epi) {
  constexpr int LD = 68;
  float(*As)[LD] = reinterpret_cast<float(*)[LD]>(sm);
  float(*Bs)[LD] = reinterpret_cast<float(*)[LD]>(sm + 16 * LD);
  const int tid = threadIdx.x, ty = tid >> 4, tx = tid & 15;
  const int lr = tid & 63, lq = tid >> 6;   // loader: row lr of the tile, k quad lq of the slab
  const bool arow_ok = m0 + lr < M, brow_ok = n0 + lr < N;
  const float* ap = A + (int64_t)(arow_ok ? arow(m0 + lr) : 0) * lda + 4 * lq;
  const float* bp = B + (int64_t)(brow_ok ? n0 + lr : 0) * K + 4 * lq;
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
  auto lda4 = [&](int k0) {
    if (!arow_ok || k0 + 4 * lq >= kend) return z4;
    float4 v;
    asm volatile("ld.global.ca.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(ap + k0));
    return v;
  };
  auto ldb4 = [&](int k0) {
    return (!brow_ok || k0 + 4 * lq >= kend) ? z4 : __ldg(reinterpret_cast<const float4*>(bp + k0));
  };
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

// the tiles of one GEMM, task t0.. of a shared task space: 64 x 64 tiles when they fill half the grid.
// Otherwise (the small-M blocks: 196 or 49 pixels) split K over 64 x 64 tiles when an fp32 accumulator
// is given -- 4 x 4 outputs per thread instead of the 2 x 2 of 32 x 32 tiles, half the shared-memory
// traffic per FMA -- the splits add into acc (atomics) and the last split of a tile (per-tile arrival
// counter) runs the epilogue and clears acc / its counter for the next launch; else 32 x 32 tiles.
// Returns the number of tasks it has.
template <class Row, class Epi>
__device__ __forceinline__ int gemm_tasks(const float* A, int lda, Row arow, const float* B, int M, int N, int K,
                                          int t0, float* sm, Epi epi, float* acc = nullptr, unsigned* cnt = nullptr) {
  const int tn64 = (N + 63) / 64, t64 = ((M + 63) / 64) * tn64;
  const bool big = 2 * t64 >= (int)gridDim.x;
  if (!big && acc && K >= 256) {
    const int sp = max(1, min((int)gridDim.x / t64, K / 128));
    const int kper = ((K + sp - 1) / sp + 15) / 16 * 16, nt = t64 * sp;
    __shared__ int last;
    for (int t = (int)blockIdx.x - t0; t < nt; t += gridDim.x) {
      if (t < 0) continue;
      const int tile_id = t / sp, ks = (t % sp) * kper;
      const int m0 = (tile_id / tn64) * 64, n0 = (tile_id % tn64) * 64;
      tile64(A, lda, arow, B, M, N, K, ks, min(K, ks + kper), m0, n0, sm,
                   [&](int m, int n, float v) { atomicAdd(acc + (int64_t)m * N + n, v); });
      __threadfence();
      __syncthreads();
      if (threadIdx.x == 0) last = atomicAdd(cnt + tile_id, 1u) == (unsigned)sp - 1;
      __syncthreads();
      if (last) {
        __threadfence();
        for (int e = threadIdx.x; e < 64 * 64; e += RX_THREADS) {
          const int m = m0 + e / 64, n = n0 + e % 64;
          if (m < M && n < N) {
            float* pa = acc + (int64_t)m * N + n;
            const float v = __ldcg(pa);
            *pa = 0.f;
            epi(m, n, v);
          }
        }
        if (threadIdx.x == 0) cnt[tile_id] = 0u;
      }
    }
    return nt;
  }
  const int bm = big ? 64 : 32, tn = (N + bm - 1) / bm, nt = ((M + bm - 1) / bm) * tn;
  for (int t = (int)blockIdx.x - t0; t < nt; t += gridDim.x) {
    if (t < 0) continue;
    if (big) tile64(A, lda, arow, B, M, N, K, 0, K, (t / tn) * 64, (t % tn) * 64, sm, epi);
    else tile<32, 32>(A, lda, arow, B, M, N, K, 0, K, (t / tn) * 32, (t % tn) * 32, sm, epi);
  }
  return nt;
}

template <int CG>   // channels per group (0: any, loops not unrolled)
__global__ void __launch_bounds__(RX_THREADS, 1) resnext_kernel(const __grid_constant__ RxParams P) {
  __shared__ __align__(16) float tsm[2 * 16 * 68];   // GEMM operand slabs
  const int tid = threadIdx.x;
  const int H = P.H, w = P.w, s = P.stride, cout = P.cout, cin = P.cin;
  const int HW = H * H, Ho = H / s, HWo = Ho * Ho;
  const int cg = CG ? CG : w / P.G;
  auto ident = [](int m) { return m; };

  stamp(P, 0);
  // ---- 1: 1x1 convolution (+ BN + ReLU), and the projection shortcut into y (its tasks continue the
  // task numbering so the two GEMMs share the grid)
  const int n1 = gemm_tasks(P.x, cin, ident, P.W1, HW, w, cin, 0, tsm, [&](int m, int n, float v) {
    P.a[(int64_t)m * w + n] = fmaxf(v * __ldg(P.s1 + n) + __ldg(P.b1 + n), 0.f);
  }, P.acc1, P.cnt);
  if (P.Wd) {
    auto srow = [&](int m) { return (m / Ho) * s * H + (m % Ho) * s; };   // output pixel -> input row
    gemm_tasks(P.x, cin, srow, P.Wd, HWo, cout, cin, n1 % (int)gridDim.x, tsm, [&](int m, int n, float v) {
      P.y[(int64_t)m * cout + n] = v * __ldg(P.sd + n) + __ldg(P.bd + n);
    }, P.acc2, P.cnt + RX_MAX_TILES);
  }
  stamp(P, 1);
  grid_sync(P, 0);
  // ---- 2 (cg >= 8): one thread per (pixel, output channel), consecutive threads = consecutive
  // channels; the quad mapping below measured slower here (fewer threads, 4x the weight loads each)
  if constexpr (CG != 4) {
    const int64_t total = (int64_t)HWo * w;
    for (int64_t idx = (int64_t)blockIdx.x * RX_THREADS + tid; idx < total; idx += (int64_t)gridDim.x * RX_THREADS) {
      const int q = (int)(idx / w), o = (int)(idx % w);
      const int g = o / cg, oo = o % cg;
      const int hs = (q / Ho) * s, ws = (q % Ho) * s;   // the pixel in the stride-1 grid
      float acc = 0.f;
#pragma unroll
      for (int t = 0; t < RX_TAPS; ++t) {
        const int i = t / 3, j = t % 3;
        const int hh = (hs + i - 1 + H) % H, ww = (ws + j - 1 + H) % H;
        const float* ar = P.a + (int64_t)(hh * H + ww) * w + g * cg;
        const float* wr = P.W2[t] + ((int64_t)g * cg + oo) * cg;
        float part = 0.f;
#pragma unroll 4
        for (int ii = 0; ii < cg; ii += 4) {
          const float4 av = ld_ca4(ar + ii);
          const float4 wv = __ldg(reinterpret_cast<const float4*>(wr + ii));
          part = fmaf(av.x, wv.x, fmaf(av.y, wv.y, fmaf(av.z, wv.z, fmaf(av.w, wv.w, part))));
        }
        if (P.m[t]) part *= __ldg(P.m[t] + hs * H + ws);
        acc += part;
      }
      P.d[idx] = fmaxf(acc * __ldg(P.s2 + o) + __ldg(P.b2 + o), 0.f);
    }
  } else
  // ---- 2 (cg == 4): grouped 3x3 convolution (+ BN + ReLU) at the strided output pixels: a thread
  // computes the 4 output channels of one group (its tap reads of a -- cg channels per tap, float4 -- are
  // shared by the 4 outputs, 4 independent accumulation chains); consecutive threads = consecutive
  // channel quads of a pixel (coalesced float4 stores of d)
  {
    const int wq = w / 4;
    const int64_t total = (int64_t)HWo * wq;
    for (int64_t idx = (int64_t)blockIdx.x * RX_THREADS + tid; idx < total; idx += (int64_t)gridDim.x * RX_THREADS) {
      const int q = (int)(idx / wq), o0 = 4 * (int)(idx % wq);
      const int g = o0 / cg, oo = o0 % cg;
      const int hs = (q / Ho) * s, ws = (q % Ho) * s;   // the pixel in the stride-1 grid
      float acc[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
      for (int t = 0; t < RX_TAPS; ++t) {
        const int i = t / 3, j = t % 3;
        const int hh = (hs + i - 1 + H) % H, ww = (ws + j - 1 + H) % H;
        const float* ar = P.a + (int64_t)(hh * H + ww) * w + g * cg;
        const float* wr = P.W2[t] + ((int64_t)g * cg + oo) * cg;
        float part[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll 4
        for (int ii = 0; ii < cg; ii += 4) {
          const float4 av = ld_ca4(ar + ii);
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const float4 wv = __ldg(reinterpret_cast<const float4*>(wr + u * cg + ii));
            part[u] = fmaf(av.x, wv.x, fmaf(av.y, wv.y, fmaf(av.z, wv.z, fmaf(av.w, wv.w, part[u]))));
          }
        }
        const float mk = P.m[t] ? __ldg(P.m[t] + hs * H + ws) : 1.f;
#pragma unroll
        for (int u = 0; u < 4; ++u) acc[u] = fmaf(part[u], mk, acc[u]);
      }
      const float4 sc = __ldg(reinterpret_cast<const float4*>(P.s2 + o0));
      const float4 bi = __ldg(reinterpret_cast<const float4*>(P.b2 + o0));
      *reinterpret_cast<float4*>(P.d + (int64_t)q * w + o0) =
          make_float4(fmaxf(acc[0] * sc.x + bi.x, 0.f), fmaxf(acc[1] * sc.y + bi.y, 0.f), fmaxf(acc[2] * sc.z + bi.z, 0.f),
                      fmaxf(acc[3] * sc.w + bi.w, 0.f));
    }
  }
  stamp(P, 2);
  grid_sync(P, 1);
  // ---- 3: 1x1 convolution (+ BN) + shortcut + ReLU
  gemm_tasks(P.d, w, ident, P.W3, HWo, cout, w, 0, tsm, [&](int m, int n, float v) {
    const int64_t o = (int64_t)m * cout + n;
    const float sc = P.Wd ? P.y[o] : __ldg(P.x + o);
    P.y[o] = fmaxf(v * __ldg(P.s3 + n) + __ldg(P.b3 + n) + sc, 0.f);
  }, P.acc3, P.cnt + 2 * RX_MAX_TILES);
  stamp(P, 3);
  // ---- exit: the last CTA resets the barrier counters for the next launch
  __syncthreads();
  __shared__ int last;
  if (tid == 0) {
    __threadfence();
    last = atomicAdd(&P.ctrl[4], 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (last && tid == 0) {
    __threadfence();
    P.ctrl[0] = P.ctrl[1] = P.ctrl[4] = 0u;
    __threadfence();
  }
}

}  // namespace rx

cudaError_t resnext_launch(const RxParams& prm, int grid, cudaStream_t s) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(RX_THREADS);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;   // the grid barriers need every CTA co-resident
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  const int cg = prm.w / prm.G;
  void (*fn)(RxParams) = cg == 4 ? rx::resnext_kernel<4> : cg == 8 ? rx::resnext_kernel<8>
                       : cg == 16 ? rx::resnext_kernel<16> : cg == 32 ? rx::resnext_kernel<32> : rx::resnext_kernel<0>;
  return cudaLaunchKernelEx(&cfg, fn, prm);
}

}  // namespace souffle
