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
#include <algorithm>
#include <cstdio>
#include <cstdlib>
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

// phases 2-4 (gates softmax, mixtures, towers) on the fused GEMM's output o1 [B][R] in shared memory;
// Wt / Wo are staged in their storage dtype (f32: fp32, else bf16)
__device__ __forceinline__ void mmoe_tail(const MmoeParams& P, float* o1, float* f, float* h1, const char* Wt,
                                          const char* Wo, const float* bt, const float* bo, bool f32, bool dbg,
                                          long long* tk) {
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, nthr = blockDim.x;
  const int B = P.B, E = P.E, De = P.De, T = P.T, Th = P.Th;
  const int R = E * De + T * E;
  // ---- 2: per-task softmax over the experts (in place, max-subtracted): warp (b, k), lane = expert
  if (warp < B * T) {
    const int b = warp / T, k = warp % T;
    float* g = o1 + b * R + E * De + k * E;
    const float v = lane < E ? g[lane] : -INFINITY;
    float m = v;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, off));
    const float ex = lane < E ? expf(v - m) : 0.f;
    float z = ex;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) z += __shfl_xor_sync(0xffffffffu, z, off);
    if (lane < E) g[lane] = ex / z;
  }
  __syncthreads();
  // ---- 3: mixtures f_k = sum_e g_k[e] * E_e (the graph's add chain, in expert order)
  for (int i = tid; i < B * T * De; i += nthr) {
    const int b = i / (T * De), k = (i / De) % T, j = i % De;
    const float* g = o1 + b * R + E * De + k * E;
    float acc = g[0] * o1[b * R + j];
#pragma unroll 4
    for (int e = 1; e < E; ++e) acc = acc + g[e] * o1[b * R + e * De + j];
    f[i] = acc;
  }
  __syncthreads();
  if (dbg && tid == 0) tk[4] = clock64();
  // ---- 4: towers: 8 lanes per hidden unit (products split over De, shuffle sum)
  for (int base = warp * 32; base < B * T * Th * 8; base += nthr) {   // warp-uniform trip count
    const int i0 = base + lane, i = i0 >> 3, part = i0 & 7;
    const bool valid = i0 < B * T * Th * 8;
    const int b = i / (T * Th), k = (i / Th) % T, r = i % Th;
    float s = 0.f;
    if (valid)
#pragma unroll 4
      for (int j = part; j < De; j += 8) s = fmaf(f[(b * T + k) * De + j], wsm(Wt, (k * Th + r) * De + j, f32), s);
    s += __shfl_xor_sync(0xffffffffu, s, 4);
    s += __shfl_xor_sync(0xffffffffu, s, 2);
    s += __shfl_xor_sync(0xffffffffu, s, 1);
    if (valid && part == 0) h1[i] = fmaxf(s + bt[k * Th + r], 0.f);
  }
  __syncthreads();
  if (warp < B * T) {
    const int b = warp / T, k = warp % T;
    float s = lane < Th ? h1[(b * T + k) * Th + lane] * wsm(Wo, k * Th + lane, f32) : 0.f;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
#pragma unroll
    for (int kk = 0; kk < MMOE_MAX_T; ++kk)
      if (kk == k && lane == 0) P.y[kk][b] = s + bo[k];
  }
}

__global__ void __launch_bounds__(MMOE_THREADS, 1) mmoe_kernel(const __grid_constant__ MmoeParams P) {
  extern __shared__ __align__(128) char smraw[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int B = P.B, D = P.D, E = P.E, De = P.De, T = P.T, Th = P.Th;
  const bool f32 = P.w_f32 != 0;
  const int es = f32 ? 4 : 2;
  const int R = E * De + T * E;               // rows of the horizontally fused GEMM
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

  long long tk[7];
  const bool dbg = P.pad != 0;   // debug timeline (SOUFFLE_MMOE_DEBUG): thread 0 prints phase times
  if (dbg && tid == 0) tk[0] = clock64();
  // ---- every parameter into shared memory with plain loads by all 1024 threads, all in flight at
  // once (one L2 round trip).  Thread 0 first writes a segment table (source, destination, length)
  // -- 16-byte weight segments and 4-byte vector segments -- then every thread loads its (up to 4 +
  // 1) elements of the concatenation before storing any (14 serial bulk-copy issues measured ~7 us,
  // per-segment load/store loops ~11 us).
  constexpr int kSeg = MMOE_SEG;
  __shared__ const char* s_src[2][kSeg];
  __shared__ char* s_dst[2][kSeg];
  __shared__ int s_pre[2][kSeg];
  __shared__ int s_nseg[2];
  // the segment table (weights: We[0..E) then per task Wg, Wt, Wo; vectors: x, be[0..E) then per task
  // bg, bt, bo) was laid out on the host at workspace initialisation: one coalesced load per entry
  if (tid < 2 * kSeg) {
    const int t = tid / kSeg, j = tid % kSeg;
    if (j <= P.nseg[t]) {
      const uint4 e = __ldg(P.seg + tid);
      s_src[t][j] = reinterpret_cast<const char*>(((unsigned long long)e.y << 32) | e.x);
      s_dst[t][j] = smraw + e.z;
      s_pre[t][j] = (int)e.w;
    }
    if (j == 0) s_nseg[t] = P.nseg[t];
  }
  __syncthreads();
  if (dbg && tid == 0) tk[2] = clock64();   // segment table built
  {
    constexpr int kW = 4;   // 16-byte units per thread (the MMoE parameters are <= 4 x 1024 x 16 B)
    uint4 wv[kW];
    int ws[kW], wo[kW];
    float fv;
    int fs = -1, fo = 0;
    int sg = 0;   // segment of the previous unit: the units of a thread ascend, so the scan resumes
#pragma unroll
    for (int j = 0; j < kW; ++j) {
      const int idx = tid + j * MMOE_THREADS;
      ws[j] = -1;
      if (idx < s_pre[0][s_nseg[0]]) {
        while (s_pre[0][sg + 1] <= idx) ++sg;
        ws[j] = sg;
        wo[j] = idx - s_pre[0][sg];
        wv[j] = __ldg(reinterpret_cast<const uint4*>(s_src[0][sg]) + wo[j]);
      }
    }
    if (tid < s_pre[1][s_nseg[1]]) {   // vectors: at most one fp32 per thread
      int sg = 0;
      while (s_pre[1][sg + 1] <= tid) ++sg;
      fs = sg;
      fo = tid - s_pre[1][sg];
      fv = __ldg(reinterpret_cast<const float*>(s_src[1][sg]) + fo);
    }
#pragma unroll
    for (int j = 0; j < kW; ++j)
      if (ws[j] >= 0) reinterpret_cast<uint4*>(s_dst[0][ws[j]])[wo[j]] = wv[j];
    if (fs >= 0) reinterpret_cast<float*>(s_dst[1][fs])[fo] = fv;
  }
  __syncthreads();
  if (dbg && tid == 0) tk[1] = clock64();
  // ---- 1: fused expert + gate GEMM, 4 threads per (row, batch) output, k interleaved by 4 (the 8
  // outputs of a warp hit 32 distinct banks: row stride D = 100 floats = 4 banks), 2 shuffles
  for (int base = warp * 32; base < 4 * R * B; base += MMOE_THREADS) {   // warp-uniform trip count
    const int it = base + lane, o = it >> 2, part = it & 3;
    const bool valid = o < R * B;
    const int r = valid ? o % R : 0, b = valid ? o / R : 0;
    const float* xr = xs + b * D;
    float s = 0.f;
    if (valid)
#pragma unroll 8
      for (int k = part; k < D; k += 4) s = fmaf(xr[k], wsm(W1, r * D + k, f32), s);
    s += __shfl_xor_sync(0xffffffffu, s, 1);
    s += __shfl_xor_sync(0xffffffffu, s, 2);
    if (valid && part == 0) {
      const float v = s + b1[r];
      o1[b * R + r] = r < E * De ? fmaxf(v, 0.f) : v;
    }
  }
  __syncthreads();
  if (dbg && tid == 0) tk[3] = clock64();
  mmoe_tail(P, o1, f, h1, Wt, Wo, bt, bo, f32, dbg, tk);
  if (dbg && tid == 0) {
    tk[5] = clock64();
    printf("mmoe clocks: segment table %lld | parameter loads %lld | gemm %lld | softmax+mix %lld | towers %lld\n",
           tk[2] - tk[0], tk[1] - tk[2], tk[3] - tk[1], tk[4] - tk[3], tk[5] - tk[4]);
  }
}

// ---------------------------------------------------------------------------------------------
// Cluster variant (B * R <= 256 fused-GEMM rows, D <= 128): the parameter fetch is the kernel's
// critical path (~59 KB through ONE SM's load path took ~1.3 us), so a cluster of MMOE_CL CTAs splits
// the horizontally fused expert + gate GEMM by rows: warp (b, r) of CTA c streams row r of its
// expert / gate weight matrix straight from global memory (coalesced, every load in flight), dots it
// with x, and writes the activated value into CTA 0's shared memory over DSMEM.  One cluster barrier
// later CTA 0 runs the softmax / mixture / tower phases (its tower parameters were fetched meanwhile).
__global__ void __launch_bounds__(1024, 1) mmoe_cluster_kernel(const __grid_constant__ MmoeParams P) {
  extern __shared__ __align__(16) float csm[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, nw = blockDim.x >> 5;
  const int B = P.B, D = P.D, E = P.E, De = P.De, T = P.T, Th = P.Th;
  const bool f32 = P.w_f32 != 0;
  const int R = E * De + T * E;
  const uint32_t cta = ptx::cluster_ctarank();
  float* o1 = csm;                          // [B][R]   (CTA 0)
  float* f = o1 + B * R;                    // [B][T][De]
  float* h1 = f + B * T * De;               // [B][T][Th]
  float* Wt = h1 + B * T * Th;              // [T][Th][De] fp32
  float* Wo = Wt + T * Th * De;             // [T][Th]
  float* bt = Wo + T * Th;                  // [T][Th]
  float* bo = bt + T * Th;                  // [T]
  // ---- this warp's fused-GEMM row: loads first (weights row, x, bias), then the dot product
  const int item = (int)cta * nw + warp;
  float s = 0.f, bias = 0.f;
  bool relu = false;
  if (item < B * R) {
    const int b = item / R, r = item % R;
    const void* w;
    if (r < E * De) {
      w = (const char*)P.We[r / De] + (int64_t)(r % De) * D * (f32 ? 4 : 2);
      bias = __ldg(P.be[r / De] + r % De);
      relu = true;
    } else {
      const int k = (r - E * De) / E, j = (r - E * De) % E;
      w = (const char*)P.Wg[k] + (int64_t)j * D * (f32 ? 4 : 2);
      bias = __ldg(P.bg[k] + j);
    }
    float wv[4], xv[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int k = lane + 32 * i;
      wv[i] = k < D ? ldw(w, k, f32) : 0.f;
      xv[i] = k < D ? __ldg(P.x + (int64_t)b * D + k) : 0.f;
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) s = fmaf(wv[i], xv[i], s);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
  }
  // ---- CTA 0: tower parameters -> shared memory (fp32), in flight with the GEMM rows
  if (cta == 0) {
    for (int i = tid; i < T * Th * De; i += blockDim.x) Wt[i] = ldw(P.Wt[i / (Th * De)], i % (Th * De), f32);
    for (int i = tid; i < T * Th; i += blockDim.x) {
      Wo[i] = ldw(P.Wo[i / Th], i % Th, f32);
      bt[i] = __ldg(P.bt[i / Th] + i % Th);
    }
    for (int i = tid; i < T; i += blockDim.x) bo[i] = __ldg(P.bo[i]);
  }
  if (item < B * R && lane == 0) {
    const float v = relu ? fmaxf(s + bias, 0.f) : s + bias;
    const uint32_t dst = ptx::mapa(ptx::smem_u32(o1 + item), 0u);   // CTA 0's o1[b][r] (item = b R + r)
    asm volatile("st.shared::cluster.f32 [%0], %1;" ::"r"(dst), "f"(v) : "memory");
  }
  // the DSMEM stores (release) -> CTA 0's reads (acquire); CTA 0's own smem writes via the barrier too
  asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
  asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (cta != 0) return;
  long long tk[7];
  mmoe_tail(P, o1, f, h1, reinterpret_cast<const char*>(Wt), reinterpret_cast<const char*>(Wo), bt, bo, true, false,
            tk);
}

}  // namespace mmoe

size_t mmoe_cluster_smem_bytes(int B, int E, int De, int T, int Th) {
  const int64_t R = (int64_t)E * De + (int64_t)T * E;
  return 4 * (size_t)(B * R + B * T * De + B * T * Th + T * Th * De + 2 * T * Th + T);
}
bool mmoe_cluster_ok(int B, int D, int E, int De, int T) {
  const int64_t R = (int64_t)E * De + (int64_t)T * E;
  return B * R <= MMOE_CL * 32 && D <= 128 && B * T <= 32 && !std::getenv("SOUFFLE_MMOE_SINGLE");
}

size_t mmoe_smem_bytes(int B, int D, int E, int De, int T, int Th) {   // (fp32 weights: upper bound)
  const int64_t R = (int64_t)E * De + (int64_t)T * E;
  return 4 * (size_t)(R * D + T * Th * De + T * Th + 12 + B * D + R + T * Th + T + B * R + B * T * De + B * T * Th);
}

cudaError_t mmoe_launch(const MmoeParams& prm, cudaStream_t s) {
  if (mmoe_cluster_ok(prm.B, prm.D, prm.E, prm.De, prm.T)) {
    const int R = prm.E * prm.De + prm.T * prm.E;
    const int warps = (prm.B * R + MMOE_CL - 1) / MMOE_CL;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(MMOE_CL);
    cfg.blockDim = dim3(32 * std::max(warps, prm.B * prm.T));
    cfg.dynamicSmemBytes = mmoe_cluster_smem_bytes(prm.B, prm.E, prm.De, prm.T, prm.Th);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = MMOE_CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, mmoe::mmoe_cluster_kernel, prm);
  }
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
