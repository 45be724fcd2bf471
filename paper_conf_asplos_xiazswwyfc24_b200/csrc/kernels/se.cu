// EfficientNet squeeze-and-excitation sub-module (M0-M9) as ONE persistent kernel on sm_100a
// (Fig. 5(c)/(d), Fig. 6):
//
//   CTA (rb, cb) owns the x tile [rows of row block rb] x [channels of channel block cb]
//   1  load the tile (16-byte loads; kept in shared memory when `reuse`), channel sums over its rows
//      -> part[rb][c]                                                        | grid barrier
//   2  pooled[c] = sum_rb part[rb][c] / HW  (thread per channel, fixed order) | grid barrier
//   3  h[s] = silu(W1[s] . pooled + b1[s])  (warp per squeeze channel)        | grid barrier
//   4  g[c] = sigmoid(W2[c] . h + b2[c]) for the CTA's channels, y = x * g for its tile (from
//      shared memory with `reuse` -- Fig. 5(d) "data reuse" -- else re-read from global: Fig. 5(c))
//
// The pool is a one-relies-on-many dependency (§5.2) and the rescale needs every pooled channel, so
// three global synchronisations are the minimum; everything else stays in one launch.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../se_types.h"
#include "ptx.cuh"

namespace souffle {
namespace se {

__device__ __forceinline__ void grid_sync(const SeParams& P, int k) {
  __syncthreads();
  if (threadIdx.x == 0) {
    ptx::red_release_add(&P.ctrl[k], 1u);
    while (ptx::ld_acquire(&P.ctrl[k]) < gridDim.x) {
    }
  }
  __syncthreads();
}

__device__ __forceinline__ float sigm(float x) { return 1.f / (1.f + __expf(-x)); }

__global__ void __launch_bounds__(SE_THREADS, 1) se_kernel(const __grid_constant__ SeParams P) {
  extern __shared__ __align__(16) float sm[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int rb = blockIdx.x / P.ncb, cb = blockIdx.x % P.ncb;
  const int r0 = rb * P.rows, nr = max(0, min(P.rows, P.HW - r0));
  const int c0 = cb * P.cbw, CW = P.cbw, C = P.C;
  const int ng = CW / 4;                                   // float4 column groups of the tile
  float* tile = sm;                                        // [rows][CW] (reuse)
  float* red = sm + (P.reuse ? P.rows * CW : 0);           // [SE_THREADS / ng][CW] partial sums
  float* g = red + SE_THREADS * 4;                         // [CW] gates of this channel block
  // ---- 1: tile -> (shared memory), channel sums over the CTA's rows
  {
    const int rl = tid / ng, gi = tid % ng, rstep = SE_THREADS / ng;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    if (rl < rstep)
      for (int r = rl; r < nr; r += rstep) {
        const float4 v = __ldg(reinterpret_cast<const float4*>(P.x + (int64_t)(r0 + r) * C + c0) + gi);
        if (P.reuse) reinterpret_cast<float4*>(tile + r * CW)[gi] = v;
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
      }
    if (rl < rstep) reinterpret_cast<float4*>(red + rl * CW)[gi] = acc;
    __syncthreads();
    for (int c = tid; c < CW; c += SE_THREADS) {
      float s = 0.f;
      for (int k = 0; k < rstep; ++k) s += red[k * CW + c];   // fixed order: deterministic
      P.part[(int64_t)rb * C + c0 + c] = s;
    }
  }
  grid_sync(P, 0);
  // ---- 2: pooled channel means (thread per channel over the grid, row blocks in order)
  for (int c = blockIdx.x * SE_THREADS + tid; c < C; c += gridDim.x * SE_THREADS) {
    float s = 0.f;
    for (int k = 0; k < P.nrb; ++k) s += __ldcg(P.part + (int64_t)k * C + c);
    P.pooled[c] = s / (float)P.HW;
  }
  grid_sync(P, 1);
  // ---- 3: squeeze: h[s] = silu(W1[s] . pooled + b1[s]), a warp per output over the grid
  for (int s = blockIdx.x * (SE_THREADS / 32) + warp; s < P.S; s += gridDim.x * (SE_THREADS / 32)) {
    float a = 0.f;
    for (int c = lane; c < C; c += 32) a = fmaf(__ldg(P.W1 + (int64_t)s * C + c), __ldcg(P.pooled + c), a);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
    if (lane == 0) {
      const float v = a + __ldg(P.b1 + s);
      P.h[s] = v * sigm(v);
    }
  }
  grid_sync(P, 2);
  // ---- 4: excitation gates of this CTA's channels, then the rescale of its tile
  for (int c = tid; c < CW; c += SE_THREADS) {
    float a = 0.f;
    for (int s = 0; s < P.S; ++s) a = fmaf(__ldg(P.W2 + (int64_t)(c0 + c) * P.S + s), __ldcg(P.h + s), a);
    g[c] = sigm(a + __ldg(P.b2 + c0 + c));
  }
  __syncthreads();
  for (int i = tid; i < nr * ng; i += SE_THREADS) {
    const int r = i / ng, gi = i % ng;
    const float4 v = P.reuse ? reinterpret_cast<const float4*>(tile + r * CW)[gi]
                             : __ldg(reinterpret_cast<const float4*>(P.x + (int64_t)(r0 + r) * C + c0) + gi);
    const float4 gg = reinterpret_cast<const float4*>(g)[gi];
    reinterpret_cast<float4*>(P.y + (int64_t)(r0 + r) * C + c0)[gi] =
        make_float4(v.x * gg.x, v.y * gg.y, v.z * gg.z, v.w * gg.w);
  }
  // ---- exit: the last CTA resets the barrier counters for the next launch
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    if (atomicAdd(&P.ctrl[3], 1u) == gridDim.x - 1) {
      P.ctrl[0] = P.ctrl[1] = P.ctrl[2] = P.ctrl[3] = 0u;
      __threadfence();
    }
  }
}

}  // namespace se

size_t se_smem_bytes(const SeParams& p) {
  return 4 * ((size_t)(p.reuse ? p.rows * p.cbw : 0) + SE_THREADS * 4 + p.cbw);
}

cudaError_t se_launch(const SeParams& prm, int grid, cudaStream_t s) {
  const size_t smem = se_smem_bytes(prm);
  cudaError_t e = cudaFuncSetAttribute(se::se_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(SE_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;   // the grid barriers need every CTA co-resident
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, se::se_kernel, prm);
}

}  // namespace souffle
