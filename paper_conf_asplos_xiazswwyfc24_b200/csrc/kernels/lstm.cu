// Persistent wavefront LSTM kernel for sm_100a (§8.4; Fig. 7).
//
// One cooperative launch runs the whole stacked LSTM (L layers x T steps).  CTA (l, p) owns nu <= 32
// hidden units [u0, u0 + nu) of layer l (u0 = p H / NP; NP CTAs per layer, as many as the SMs allow,
// so that the per-step GEMV -- bound by reading the CTA's weights from shared memory -- is spread
// over all SMs): the 4 nu gate rows (i, f, g, o of those units) of [W_ih | W_hh] are
// loaded into shared memory ONCE and reused for all T steps (the paper's "weights stay on chip";
// HBM reads the 10.5 MB of bf16 weights once instead of once per step).  Per step:
//   wait   h(l, t-1) and h(l-1, t) are read as (value, tag) words straight from L2, spinning until
//          every tag carries this run's step (one round trip = readiness + data; no grid barrier,
//          no fence; the wavefront is L + T - 1 = 109 cells deep)
//   GEMV   gates = [W_ih | W_hh] [x_t ; h_{t-1}] on CUDA cores, bf16 (or fp32) weights x fp32
//          activations, fp32 accumulation (activations are never rounded: SURVEY §8(c))
//   cell   i, f, o = sigmoid, g = tanh; c = f c + i g; h = o tanh(c)  (torch.nn.LSTM semantics)
//   publish h(l, t) for the 32 units as (value, tag) 64-bit words
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../lstm_types.h"
#include "ptx.cuh"

namespace souffle {
namespace lstm {

// gate nonlinearities on the SFU (ex2 + rcp): the cell update is on the wavefront's critical path
// (one warp, every step); absolute error ~1e-7, far inside the fp32 parity tolerance (rel 1e-4)
__device__ __forceinline__ float sigm(float x) { return __fdividef(1.f, 1.f + __expf(-x)); }
__device__ __forceinline__ float tanh_f(float x) {
  const float t = __expf(-2.f * fabsf(x));
  return copysignf(__fdividef(1.f - t, 1.f + t), x);
}

// 8 consecutive weights of row r (smem) as fp32
template <bool F32>
__device__ __forceinline__ void wload8(const char* w, int K, int r, int g, float* o) {
  if constexpr (F32) {
    const float4* p = reinterpret_cast<const float4*>(w) + ((int64_t)r * K + 8 * g) / 4;
    const float4 a = p[0], b = p[1];
    o[0] = a.x; o[1] = a.y; o[2] = a.z; o[3] = a.w; o[4] = b.x; o[5] = b.y; o[6] = b.z; o[7] = b.w;
  } else {
    const uint4 a = *reinterpret_cast<const uint4*>(reinterpret_cast<const uint16_t*>(w) + (int64_t)r * K + 8 * g);
    const uint32_t u[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      o[2 * j] = __uint_as_float(u[j] << 16);
      o[2 * j + 1] = __uint_as_float(u[j] & 0xFFFF0000u);
    }
  }
}

template <bool F32>
__global__ void __launch_bounds__(LSTM_THREADS, 1) lstm_kernel(const __grid_constant__ LstmParams P) {
  extern __shared__ __align__(16) char smem[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int l = blockIdx.x / P.NP, p = blockIdx.x % P.NP;
  const int H = P.H, T = P.T, NP = P.NP, Kst = P.K_max;
  const int u0 = (p * H) / NP, nu = ((p + 1) * H) / NP - u0;   // this CTA's hidden units (nu <= 32)
  const int R = 4 * nu;                                         // gate rows r = gate * nu + j
  const LstmLayer& Ly = P.layers[l];
  const int I = Ly.in_dim, K = I + H;
  constexpr int ES = F32 ? 4 : 2;
  char* w = smem;                                                        // [128][Kst] weights
  float* xh = reinterpret_cast<float*>(smem + (size_t)LSTM_ROWS * Kst * ES);   // [Kst]  [x_t ; h_{t-1}]
  float* gates = xh + Kst;                                               // [128]
  float* bias = gates + LSTM_ROWS;                                       // [128] b_ih + b_hh

  // ---- weights of this CTA's 128 gate rows -> shared memory (once for all T steps)
  {
    const int vpr = K * ES / 16;   // 16-byte vectors per row
    for (int e = tid; e < LSTM_ROWS * vpr; e += LSTM_THREADS) {
      const int r = e / vpr, v = e % vpr;
      if (r >= R) break;
      const int grow = (r / nu) * H + u0 + (r % nu);
      const int col = v * 16 / ES;   // first element of this vector
      const char* src = col < I ? (const char*)Ly.W + ((int64_t)grow * I + col) * ES
                                : (const char*)Ly.U + ((int64_t)grow * H + (col - I)) * ES;
      // asynchronous copies: every chunk of the tile in flight at once (a load -> store loop waited for
      // each round trip in turn: ~10 us before the first step)
      ptx::cp_async16(w + ((int64_t)r * Kst + col) * ES, src);
    }
    ptx::cp_async_wait_all();
    for (int r = tid; r < R; r += LSTM_THREADS) {
      const int grow = (r / nu) * H + u0 + (r % nu);
      bias[r] = __ldg(Ly.b_ih + grow) + __ldg(Ly.b_hh + grow);
    }
  }
  const int unit = u0 + lane;
  const bool own = lane < nu;
  float c = (warp == 0 && own) ? __ldg(Ly.c0 + unit) : 0.f;
  float h = 0.f;
  __syncthreads();

  auto stamp = [&](int t, int k) {   // debug timeline: SM clock cycles (%globaltimer ticks in 256 ns steps)
    if (P.prof && blockIdx.x == P.prof_cta && tid == 0) P.prof[4 * t + k] = (unsigned long long)clock64();
  };
  // [x_t ; h_{t-1}] is kept split: elements 8g..8g+3 at float4 g, 8g+4..8g+7 at float4 K/8 + g, so the
  // GEMV lanes (consecutive g) read consecutive float4s (the interleaved layout was 2-way bank-conflicted)
  const int khalf = K / 2;
  auto xpos = [&](int k) { return ((k >> 3) << 2) + (k & 3) + ((k & 4) ? khalf : 0); };
  const unsigned gen = *(volatile unsigned*)P.gen;   // written by the previous launch's last CTA
  const unsigned tag0 = gen * (unsigned)(T + 1) + 1u;
  for (int t = 0; t < T; ++t) {
    stamp(t, 0);
    // ---- [x_t ; h_{t-1}] -> shared memory; operands produced by other CTAs are spun on until their
    // tag is this run's step (x of layer l > 0 is h(l-1, t); h is h(l, t-1))
    {
      // every operand word of this thread is requested before any is waited on (one round trip)
      constexpr int kMaxPer = 2;   // K <= 2 * LSTM_THREADS
      const uint2* src[kMaxPer];
      unsigned want[kMaxPer];
      unsigned long long w64[kMaxPer];
#pragma unroll
      for (int i = 0; i < kMaxPer; ++i) {
        const int k = tid + i * LSTM_THREADS;
        src[i] = nullptr;
        if (k >= K) continue;
        if (k < I && l == 0) {
          xh[xpos(k)] = __ldg(P.X + (int64_t)t * I + k);
        } else if (k >= I && t == 0) {
          xh[xpos(k)] = __ldg(Ly.h0 + (k - I));
        } else {
          src[i] = (k < I) ? P.hbuf + ((int64_t)(l - 1) * T + t) * H + k : P.hbuf + ((int64_t)l * T + t - 1) * H + (k - I);
          want[i] = tag0 + (unsigned)(k < I ? t : t - 1);
          asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(w64[i]) : "l"(src[i]) : "memory");
        }
      }
#pragma unroll
      for (int i = 0; i < kMaxPer; ++i) {
        if (src[i] == nullptr) continue;
        while ((unsigned)(w64[i] >> 32) != want[i])   // one single-copy-atomic word: tag in the high half
          asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(w64[i]) : "l"(src[i]) : "memory");
        xh[xpos(tid + i * LSTM_THREADS)] = __uint_as_float((unsigned)w64[i]);
      }
    }
    __syncthreads();
    stamp(t, 1);
    // ---- gates: warp w computes rows RPW*w ..; lanes split the K columns in groups of 8 (warps
    // beyond the CTA's 4 nu rows skip: the smem weight reads are the step's bound)
    if (warp * 8 < R) {
      constexpr int RPW = LSTM_ROWS / (LSTM_THREADS / 32);   // rows per warp (8 with 16 warps)
      static_assert(RPW == 8, "reduction below assumes 8 rows per warp");
      float acc[RPW];
#pragma unroll
      for (int i = 0; i < RPW; ++i) acc[i] = 0.f;
      const int ng = K / 8;
      for (int g = lane; g < ng; g += 32) {
        const float4 xa = *reinterpret_cast<const float4*>(xh + 4 * g);
        const float4 xb = *reinterpret_cast<const float4*>(xh + khalf + 4 * g);
        const float xv[8] = {xa.x, xa.y, xa.z, xa.w, xb.x, xb.y, xb.z, xb.w};
        float wv[RPW][8];
#pragma unroll
        for (int i = 0; i < RPW; ++i) wload8<F32>(w, Kst, warp * RPW + i, g, wv[i]);
#pragma unroll
        for (int i = 0; i < RPW; ++i)
#pragma unroll
          for (int e = 0; e < 8; ++e) acc[i] = fmaf(wv[i][e], xv[e], acc[i]);
      }
      // transpose-reduce 8 row sums over the 32 lanes (4 + 2 + 1 + 2 shuffles)
      float v4[4];
      const bool b4 = lane & 16;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float send = b4 ? acc[i] : acc[i + 4];
        const float keep = b4 ? acc[i + 4] : acc[i];
        v4[i] = keep + __shfl_xor_sync(0xffffffffu, send, 16);
      }
      float v2[2];
      const bool b3 = lane & 8;
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        const float send = b3 ? v4[i] : v4[i + 2];
        const float keep = b3 ? v4[i + 2] : v4[i];
        v2[i] = keep + __shfl_xor_sync(0xffffffffu, send, 8);
      }
      const bool b2 = lane & 4;
      float v1 = (b2 ? v2[1] : v2[0]) + __shfl_xor_sync(0xffffffffu, b2 ? v2[0] : v2[1], 4);
      v1 += __shfl_xor_sync(0xffffffffu, v1, 2);
      v1 += __shfl_xor_sync(0xffffffffu, v1, 1);
      const int r = 4 * ((lane >> 4) & 1) + 2 * ((lane >> 3) & 1) + ((lane >> 2) & 1);
      if ((lane & 3) == 0) gates[warp * RPW + r] = v1;
    }
    __syncthreads();
    stamp(t, 2);
    // ---- cell update (warp 0, one unit per lane) and publication of h(l, t)
    if (warp == 0 && own) {
      const float gi = gates[lane] + bias[lane];
      const float gf = gates[nu + lane] + bias[nu + lane];
      const float gg = gates[2 * nu + lane] + bias[2 * nu + lane];
      const float go = gates[3 * nu + lane] + bias[3 * nu + lane];
      c = sigm(gf) * c + sigm(gi) * tanh_f(gg);
      h = sigm(go) * tanh_f(c);
      if (l == P.L - 1) P.top[t][unit] = h;
      const unsigned long long w64 = ((unsigned long long)(tag0 + (unsigned)t) << 32) | __float_as_uint(h);
      uint2* dst = P.hbuf + ((int64_t)l * T + t) * H + unit;
      asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(dst), "l"(w64) : "memory");
    }
    stamp(t, 3);
  }
  if (warp == 0 && own) {
    Ly.h_n[unit] = h;
    Ly.c_n[unit] = c;
  }
  // ---- exit: the last CTA advances the run generation (tags of the next launch differ)
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    const unsigned old = atomicAdd(P.gen + 1, 1u);
    if (old == gridDim.x - 1) {
      P.gen[1] = 0u;
      P.gen[0] = gen + 1u;
      __threadfence();
    }
  }
}

// ---------------------------------------------------------------------------------------------
// Register-resident variant (K = I + H <= 512 and <= 20 units per CTA, e.g. the 10 x 256 x 100
// configuration at 14 CTAs per layer): the CTA's 4 nu gate rows are held in fp32 REGISTERS for all
// T steps (80 weights per thread: 4 nu x 512 x 4 B = 152 KB of the 256 KB register file), so a
// step's GEMV reads only the 2 KB operand vector from shared memory and issues packed FFMA2s.
// Warp w owns rows j = 5 (w % 4) + i (i < 5) of gate w / 4; lane q owns columns
// k = 4 (q + 32 c) + e (c < 4, e < 4: consecutive lanes read consecutive float4s of [x; h], no bank
// conflicts); the warp's 32 partial sums of each row are combined by a 5-level transpose reduction
// (8 shuffles), so no cross-warp reduction is needed.  Same dependency protocol and cell as above.
template <bool F32>
__global__ void __launch_bounds__(LSTM_THREADS, 1) lstm_reg_kernel(const __grid_constant__ LstmParams P) {
  __shared__ __align__(16) float xh[LSTM_REG_K];   // [x_t ; h_{t-1}], zero beyond K
  __shared__ float gates[LSTM_ROWS];
  __shared__ float bias[LSTM_ROWS];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int l = blockIdx.x / P.NP, p = blockIdx.x % P.NP;
  const int H = P.H, T = P.T, NP = P.NP;
  const int u0 = (p * H) / NP, nu = ((p + 1) * H) / NP - u0;   // nu <= 20
  const LstmLayer& Ly = P.layers[l];
  const int I = Ly.in_dim, K = I + H;
  const int gate = warp >> 2, j0 = LSTM_REG_RPW * (warp & 3);   // rows j0 .. j0 + 4 of this gate
  const bool has_rows = j0 < nu;

  // ---- this thread's 80 weights -> fp32 registers (once for all T steps); zero outside the tile.
  // I % 8 == 0, so a 4-column group never straddles W_ih | W_hh and its loads are 8 / 16-byte aligned
  float2 w[LSTM_REG_RPW][4][2];
#pragma unroll
  for (int i = 0; i < LSTM_REG_RPW; ++i) {
    const int j = j0 + i;
    const int64_t grow = (int64_t)gate * H + u0 + j;
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const int k = 4 * (lane + 32 * c);
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (j < nu && k < K) {
        const int64_t off = k < I ? grow * I + k : grow * H + (k - I);
        const void* base = k < I ? Ly.W : Ly.U;
        if constexpr (F32) {
          v = __ldg(reinterpret_cast<const float4*>(base) + off / 4);
        } else {
          const uint2 u = __ldg(reinterpret_cast<const uint2*>(base) + off / 4);
          v = make_float4(__uint_as_float(u.x << 16), __uint_as_float(u.x & 0xFFFF0000u), __uint_as_float(u.y << 16),
                          __uint_as_float(u.y & 0xFFFF0000u));
        }
      }
      w[i][c][0] = make_float2(v.x, v.y);
      w[i][c][1] = make_float2(v.z, v.w);
    }
  }
  for (int r = tid; r < 4 * nu; r += LSTM_THREADS) {
    const int grow = (r / nu) * H + u0 + (r % nu);
    bias[r] = __ldg(Ly.b_ih + grow) + __ldg(Ly.b_hh + grow);
  }
  for (int k = tid; k < LSTM_REG_K; k += LSTM_THREADS) xh[k] = 0.f;
  const int unit = u0 + lane;
  const bool own = lane < nu;
  float c = (warp == 0 && own) ? __ldg(Ly.c0 + unit) : 0.f;
  float h = 0.f;
  __syncthreads();

  auto stamp = [&](int t, int k) {
    if (P.prof && blockIdx.x == P.prof_cta && tid == 0) P.prof[4 * t + k] = (unsigned long long)clock64();
  };
  const unsigned gen = *(volatile unsigned*)P.gen;
  const unsigned tag0 = gen * (unsigned)(T + 1) + 1u;
  for (int t = 0; t < T; ++t) {
    stamp(t, 0);
    // ---- [x_t ; h_{t-1}] -> shared memory (thread k fetches element k; K <= 512 threads)
    if (tid < K) {
      const int k = tid;
      if (k < I && l == 0) {
        xh[k] = __ldg(P.X + (int64_t)t * I + k);
      } else if (k >= I && t == 0) {
        xh[k] = __ldg(Ly.h0 + (k - I));
      } else {
        const uint2* src = (k < I) ? P.hbuf + ((int64_t)(l - 1) * T + t) * H + k : P.hbuf + ((int64_t)l * T + t - 1) * H + (k - I);
        const unsigned want = tag0 + (unsigned)(k < I ? t : t - 1);
        unsigned long long w64;
        asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(w64) : "l"(src) : "memory");
        while ((unsigned)(w64 >> 32) != want)
          asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(w64) : "l"(src) : "memory");
        xh[k] = __uint_as_float((unsigned)w64);
      }
    }
    __syncthreads();
    stamp(t, 1);
    // ---- gates: 40 FFMA2 per thread, then the warp's transpose reduction of its 5 row sums
    if (has_rows) {
      const float4* x4 = reinterpret_cast<const float4*>(xh);
      float4 xv[4];
#pragma unroll
      for (int cc = 0; cc < 4; ++cc) xv[cc] = x4[lane + 32 * cc];
      float2 a[LSTM_REG_RPW];
#pragma unroll
      for (int i = 0; i < LSTM_REG_RPW; ++i) a[i] = make_float2(0.f, 0.f);
#pragma unroll
      for (int cc = 0; cc < 4; ++cc) {
        const float2 xa = make_float2(xv[cc].x, xv[cc].y), xb = make_float2(xv[cc].z, xv[cc].w);
#pragma unroll
        for (int i = 0; i < LSTM_REG_RPW; ++i) {
          a[i] = __ffma2_rn(w[i][cc][0], xa, a[i]);
          a[i] = __ffma2_rn(w[i][cc][1], xb, a[i]);
        }
      }
      float v[LSTM_REG_RPW];
#pragma unroll
      for (int i = 0; i < LSTM_REG_RPW; ++i) v[i] = a[i].x + a[i].y;
      // level 1 (xor 16): rows (0, 1, 2) | (3, 4, -); level 2 (xor 8): (u0, u1) | (u2, -);
      // level 3 (xor 4): one row; levels 4-5 (xor 2, 1): full sums.  Row = 3 b16 + 2 b8 + b4.
      const bool b16 = lane & 16, b8 = lane & 8, b4 = lane & 4;
      float u[3];
#pragma unroll
      for (int m = 0; m < 3; ++m) {
        const float lo = v[m], hi = m + 3 < LSTM_REG_RPW ? v[m + 3] : 0.f;
        u[m] = (b16 ? hi : lo) + __shfl_xor_sync(0xffffffffu, b16 ? lo : hi, 16);
      }
      float y[2];
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        const float lo = u[m], hi = m == 0 ? u[2] : 0.f;
        y[m] = (b8 ? hi : lo) + __shfl_xor_sync(0xffffffffu, b8 ? lo : hi, 8);
      }
      float z = (b4 ? y[1] : y[0]) + __shfl_xor_sync(0xffffffffu, b4 ? y[0] : y[1], 4);
      z += __shfl_xor_sync(0xffffffffu, z, 2);
      z += __shfl_xor_sync(0xffffffffu, z, 1);
      const int loc = 2 * (int)b8 + (int)b4, row = 3 * (int)b16 + loc;
      if ((lane & 3) == 0 && loc < 3 && row < LSTM_REG_RPW && j0 + row < nu) gates[gate * nu + j0 + row] = z;
    }
    __syncthreads();
    stamp(t, 2);
    // ---- cell update (warp 0, one unit per lane) and publication of h(l, t)
    if (warp == 0 && own) {
      const float gi = gates[lane] + bias[lane];
      const float gf = gates[nu + lane] + bias[nu + lane];
      const float gg = gates[2 * nu + lane] + bias[2 * nu + lane];
      const float go = gates[3 * nu + lane] + bias[3 * nu + lane];
      c = sigm(gf) * c + sigm(gi) * tanh_f(gg);
      h = sigm(go) * tanh_f(c);
      if (l == P.L - 1) P.top[t][unit] = h;
      const unsigned long long w64 = ((unsigned long long)(tag0 + (unsigned)t) << 32) | __float_as_uint(h);
      uint2* dst = P.hbuf + ((int64_t)l * T + t) * H + unit;
      asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(dst), "l"(w64) : "memory");
    }
    stamp(t, 3);
  }
  if (warp == 0 && own) {
    Ly.h_n[unit] = h;
    Ly.c_n[unit] = c;
  }
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    const unsigned old = atomicAdd(P.gen + 1, 1u);
    if (old == gridDim.x - 1) {
      P.gen[1] = 0u;
      P.gen[0] = gen + 1u;
      __threadfence();
    }
  }
}

}  // namespace lstm

size_t lstm_smem_bytes(int K_max, int w_f32) {
  return (size_t)LSTM_ROWS * K_max * (w_f32 ? 4 : 2) + (size_t)(K_max + 2 * LSTM_ROWS) * 4;
}

cudaError_t lstm_launch(const LstmParams& prm, int grid, cudaStream_t s) {
  const size_t smem = prm.reg ? 0 : lstm_smem_bytes(prm.K_max, prm.w_f32);
  void (*fn)(LstmParams) = prm.reg ? (prm.w_f32 ? lstm::lstm_reg_kernel<true> : lstm::lstm_reg_kernel<false>)
                                   : (prm.w_f32 ? lstm::lstm_kernel<true> : lstm::lstm_kernel<false>);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(LSTM_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;   // all CTAs co-resident: the flag waits require it
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, fn, prm);
}

}  // namespace souffle
