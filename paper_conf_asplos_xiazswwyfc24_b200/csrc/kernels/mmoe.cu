// Fused multi-gate mixture-of-experts kernel for sm_100a (Table 2; §6.1: the expert
// and gate GEMMs share x and are horizontally fused into one GEMM; Table 5: one kernel).
//
// At batch 1 the model is ~30 KFLOP over ~59 KB of parameters: it is launch- and latency-bound, so
// the whole TE program runs in ONE CTA with every parameter staged once into shared memory (all
// loads issued together) and the intermediate tensors (experts, gates, mixtures, tower activations)
// never leaving it:
//   1  [E_1 .. E_8 | G_1 G_2] = x [W_e1 .. W_e8 | W_g1 W_g2]^T + b   (horizontal fusion, warp per row)
//      ReLU on the expert columns
//   2  g_k = softmax(G_k)                       (max-subtracted, per task)
//   3  f_k = sum_e g_k[e] E_e                    (the slice * expert products and their sum chain)
//   4  y_k = W_o,k relu(W_t,k f_k + b_t,k) + b_o,k
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../mmoe_types.h"
#include "ptx.cuh"

namespace souffle {
namespace mmoe {

__device__ __forceinline__ float ldw(const void* p, int64_t i, bool f32) {
  if (f32) return __ldg(reinterpret_cast<const float*>(p) + i);
  const unsigned short b = __ldg(reinterpret_cast<const unsigned short*>(p) + i);
  return __uint_as_float(((uint32_t)b) << 16);
}

// weight element i of a staged tensor (raw storage dtype in shared memory)
__device__ __forceinline__ float wsm(const char* base, int64_t i, bool f32) {
  if (f32) return reinterpret_cast<const float*>(base)[i];
  return __uint_as_float(((uint32_t) reinterpret_cast<const unsigned short*>(base)[i]) << 16);
}

__global__ void __launch_bounds__(MMOE_THREADS, 1) mmoe_kernel(const __grid_constant__ MmoeParams P) {
  extern __shared__ __align__(128) char smraw[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int B = P.B, D = P.D, E = P.E, De = P.De, T = P.T, Th = P.Th;
  const bool f32 = P.w_f32 != 0;
  const int es = f32 ? 4 : 2;
  const int R = E * De + T * E;               // rows of the horizontally fused GEMM
  __shared__ __align__(8) uint64_t bar;
  // raw (storage dtype) weights, staged by bulk copies: [R][D] experts then gates, [T][Th][De], [T][Th]
  char* W1 = smraw;
  char* Wt = W1 + (((int64_t)R * D * es + 15) & ~15);
  char* Wo = Wt + (((int64_t)T * Th * De * es + 15) & ~15);
  float* xs = reinterpret_cast<float*>(Wo + (((int64_t)T * Th * es + 15) & ~15));   // [B][D]
  float* b1 = xs + B * D;                     // [R]
  float* bt = b1 + R;                         // [T][Th]
  float* bo = bt + T * Th;                    // [T]
  float* o1 = bo + T;                         // [B][R]   expert / gate pre-activations
  float* f = o1 + B * R;                      // [B][T][De]
  float* h1 = f + B * T * De;                 // [B][T][Th]

  // ---- every weight tensor in flight at once: one bulk copy (TMA engine) per tensor, one mbarrier
  if (tid == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
    const uint32_t bytes = (uint32_t)(((int64_t)E * De * D + (int64_t)T * E * D + (int64_t)T * Th * De + T * Th) * es);
    ptx::mbar_arrive_expect_tx(&bar, bytes);
    for (int e = 0; e < E; ++e)
      ptx::bulk_g2s(W1 + (int64_t)e * De * D * es, P.We[e], (uint32_t)(De * D * es), &bar);
    for (int k = 0; k < T; ++k)
      ptx::bulk_g2s(W1 + (int64_t)(E * De + k * E) * D * es, P.Wg[k], (uint32_t)(E * D * es), &bar);
    for (int k = 0; k < T; ++k) ptx::bulk_g2s(Wt + (int64_t)k * Th * De * es, P.Wt[k], (uint32_t)(Th * De * es), &bar);
    for (int k = 0; k < T; ++k) ptx::bulk_g2s(Wo + (int64_t)k * Th * es, P.Wo[k], (uint32_t)(Th * es), &bar);
  }
  for (int i = tid; i < B * D; i += MMOE_THREADS) xs[i] = __ldg(P.x + i);
  for (int r = tid; r < R; r += MMOE_THREADS)
    b1[r] = r < E * De ? __ldg(P.be[r / De] + r % De) : __ldg(P.bg[(r - E * De) / E] + (r - E * De) % E);
  for (int i = tid; i < T * Th; i += MMOE_THREADS) bt[i] = __ldg(P.bt[i / Th] + i % Th);
  for (int k = tid; k < T; k += MMOE_THREADS) bo[k] = __ldg(P.bo[k]);
  __syncthreads();   // mbarrier initialised before anyone waits on it
  ptx::mbar_wait(&bar, 0);
  // ---- 1: fused expert + gate GEMM; a warp computes 4 (row, batch) outputs at once (lanes split D,
  // four independent accumulators and shuffle trees in flight: the chain latency is paid once per 4)
  constexpr int kO = 4, kWarps = MMOE_THREADS / 32;
  for (int o0 = warp * kO; o0 < R * B; o0 += kWarps * kO) {
    float s[kO] = {0.f, 0.f, 0.f, 0.f};
    for (int k = lane; k < D; k += 32) {
#pragma unroll
      for (int j = 0; j < kO; ++j) {
        const int o = o0 + j;
        if (o < R * B) s[j] = fmaf(xs[(o / R) * D + k], wsm(W1, (int64_t)(o % R) * D + k, f32), s[j]);
      }
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1)
#pragma unroll
      for (int j = 0; j < kO; ++j) s[j] += __shfl_xor_sync(0xffffffffu, s[j], off);
    if (lane < kO && o0 + lane < R * B) {
      const int o = o0 + lane, r = o % R, b = o / R;
      const float sl = lane == 0 ? s[0] : lane == 1 ? s[1] : lane == 2 ? s[2] : s[3];
      const float v = sl + b1[r];
      o1[b * R + r] = r < E * De ? fmaxf(v, 0.f) : v;
    }
  }
  __syncthreads();
  // ---- 2: per-task softmax over the experts (in place, max-subtracted)
  if (tid < B * T) {
    const int b = tid / T, k = tid % T;
    float* g = o1 + b * R + E * De + k * E;
    float m = -INFINITY;
    for (int e = 0; e < E; ++e) m = fmaxf(m, g[e]);
    float z = 0.f;
    for (int e = 0; e < E; ++e) {
      g[e] = expf(g[e] - m);
      z += g[e];
    }
    for (int e = 0; e < E; ++e) g[e] = g[e] / z;
  }
  __syncthreads();
  // ---- 3: mixtures f_k = sum_e g_k[e] * E_e (the graph's add chain, in expert order)
  for (int i = tid; i < B * T * De; i += MMOE_THREADS) {
    const int b = i / (T * De), k = (i / De) % T, j = i % De;
    const float* g = o1 + b * R + E * De + k * E;
    float acc = g[0] * o1[b * R + j];
    for (int e = 1; e < E; ++e) acc = acc + g[e] * o1[b * R + e * De + j];
    f[i] = acc;
  }
  __syncthreads();
  // ---- 4: towers
  for (int i = tid; i < B * T * Th; i += MMOE_THREADS) {
    const int b = i / (T * Th), k = (i / Th) % T, r = i % Th;
    float s = 0.f;
    for (int j = 0; j < De; ++j) s = fmaf(f[(b * T + k) * De + j], wsm(Wt, (int64_t)(k * Th + r) * De + j, f32), s);
    h1[i] = fmaxf(s + bt[k * Th + r], 0.f);
  }
  __syncthreads();
  if (tid < B * T) {
    const int b = tid / T, k = tid % T;
    float s = 0.f;
    for (int r = 0; r < Th; ++r) s = fmaf(h1[(b * T + k) * Th + r], wsm(Wo, k * Th + r, f32), s);
    P.y[k][b] = s + bo[k];
  }
}

}  // namespace mmoe

size_t mmoe_smem_bytes(int B, int D, int E, int De, int T, int Th) {   // (fp32 weights: upper bound)
  const int64_t R = (int64_t)E * De + (int64_t)T * E;
  return 4 * (size_t)(R * D + T * Th * De + T * Th + 12 + B * D + R + T * Th + T + B * R + B * T * De + B * T * Th);
}

cudaError_t mmoe_launch(const MmoeParams& prm, cudaStream_t s) {
  const size_t smem = mmoe_smem_bytes(prm.B, prm.D, prm.E, prm.De, prm.T, prm.Th);
  static size_t set = 0;
  if (smem > set) {
    cudaError_t e = cudaFuncSetAttribute(mmoe::mmoe_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    set = smem;
  }
  mmoe::mmoe_kernel<<<1, MMOE_THREADS, smem, s>>>(prm);
  return cudaGetLastError();
}

}  // namespace souffle
