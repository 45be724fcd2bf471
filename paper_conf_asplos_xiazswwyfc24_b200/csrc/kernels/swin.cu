// Swin-Transformer pattern kernels on sm_100a (B200): the fused subprograms of a Swin block
// (Table 2), see csrc/swin_types.h for the op list.
//
//   sw_gemm_kernel  persistent tcgen05 GEMM: warp 0 streams A / W K-chunks by TMA through a ring,
//                   warp 1 issues tcgen05.mma (M = 128, N = BN <= 256, K = 16) into one of two TMEM
//                   accumulators, warps 2-5 run the fused epilogue of the previous tile meanwhile
//   sw_attn_kernel  window attention, two (window, head) units per M = 128 tile (QK^T, bias + mask,
//                   softmax in fp32 registers, PV) -- the reductions of Fig. 1(c) kept on chip
//   sw_row_kernel   LayerNorm of rows gathered through the block's quasi-affine index maps
//   sw_im2col_kernel, sw_head_kernel   patch embedding gather; final LN + mean pool + classifier
#include <cuda.h>
#include <cstdlib>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>
#include <algorithm>

#include "../swin_types.h"
#include "ptx.cuh"

namespace souffle {
namespace swin {

struct alignas(64) GemmArgs {
  CUtensorMap ta, tb;
  SwGemm g;
};
struct alignas(64) AttnArgs {
  CUtensorMap tq, tk, tv;
  SwAttn a;
};

__device__ __forceinline__ uint32_t pack_bf16(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}
__device__ __forceinline__ uint16_t bf16_bits(float a) {
  __nv_bfloat16 b = __float2bfloat16_rn(a);
  return *reinterpret_cast<uint16_t*>(&b);
}
__device__ __forceinline__ float bf2f(uint16_t b) { return __uint_as_float(((uint32_t)b) << 16); }
// erf-GELU (the TE's exact-erf semantics) with erf(t) = 1 - 2^(t P7(t)) on t = |x| <= 3.92 (erf = 1 in
// fp32 beyond): one polynomial, one MUFU.EX2, no branch (CUDA's erff takes two divergent polynomial
// paths).  |erf error| <= 3e-7 absolute (fit in DESIGN.md R19), GELU within 5e-7 absolute -- far
// below the bf16 rounding of the GELU output that follows.
__device__ __forceinline__ float gelu_erf(float x) {
  const float u = x * 0.70710678118654752f;
  const float t = fminf(fabsf(u), 3.92f);
  float p = -4.4602740672416985e-05f;
  p = fmaf(p, t, 4.394397255964577e-04f);
  p = fmaf(p, t, -1.4703732449561357e-03f);
  p = fmaf(p, t, -8.046277216635644e-04f);
  p = fmaf(p, t, 2.8278736397624016e-02f);
  p = fmaf(p, t, -0.14849244058132172f);
  p = fmaf(p, t, -0.9184142351150513f);
  p = fmaf(p, t, -1.627908706665039f);
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(t * p));
  const float e = copysignf(1.f - y, u);
  return 0.5f * x * (1.f + e);
}
// the same GELU on two values with packed fp32 arithmetic (FFMA2 / FMUL2 / FADD2): every lane's result
// is the IEEE-rounded scalar result, so the output is bit-identical to gelu_erf in half the issue
// slots (the FC1 epilogue is issue-bound: 128 x 256 GELUs per tile on 8 warps)
__device__ __forceinline__ float2 gelu_erf2(float2 x) {
  auto cc = [](float c) { return make_float2(c, c); };
  const float2 u = __fmul2_rn(x, cc(0.70710678118654752f));
  const float2 t = make_float2(fminf(fabsf(u.x), 3.92f), fminf(fabsf(u.y), 3.92f));
  float2 p = cc(-4.4602740672416985e-05f);
  p = __ffma2_rn(p, t, cc(4.394397255964577e-04f));
  p = __ffma2_rn(p, t, cc(-1.4703732449561357e-03f));
  p = __ffma2_rn(p, t, cc(-8.046277216635644e-04f));
  p = __ffma2_rn(p, t, cc(2.8278736397624016e-02f));
  p = __ffma2_rn(p, t, cc(-0.14849244058132172f));
  p = __ffma2_rn(p, t, cc(-0.9184142351150513f));
  p = __ffma2_rn(p, t, cc(-1.627908706665039f));
  const float2 tp = __fmul2_rn(t, p);
  float2 y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y.x) : "f"(tp.x));
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y.y) : "f"(tp.y));
  const float2 e = make_float2(copysignf(1.f - y.x, u.x), copysignf(1.f - y.y, u.y));
  return __fmul2_rn(__fmul2_rn(x, cc(0.5f)), __fadd2_rn(cc(1.f), e));   // (0.5 x)(1 + e) as in gelu_erf
}
__device__ __forceinline__ uint32_t pack_gelu2(float a, float b) {
  const float2 g = gelu_erf2(make_float2(a, b));
  return pack_bf16(g.x, g.y);
}
__device__ __forceinline__ uint32_t sw128(int row, int kbyte) {
  return (uint32_t)(row * 128 + ((((kbyte >> 4) ^ (row & 7)) & 7) << 4) + (kbyte & 15));
}

// programmatic dependent launch: let the next kernel of the stream start its prologue now, and wait
// for the previous kernel's completion (and memory) before touching global memory
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
// debug trace: CTA 0 stamps %globaltimer when launch `op` passes its dependency wait
__device__ __forceinline__ void trace_stamp(unsigned long long* tr, int op) {
  if (tr && blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    tr[op] = t;
  }
}
constexpr int kEpiWarps = SW_GEMM_THREADS / 32 - 2, kEpiThreads = 32 * kEpiWarps, kEpiGroups = kEpiWarps / 4;
static_assert(kEpiWarps % 4 == 0, "epilogue warps cover the 4 TMEM lane quarters evenly");
__device__ __forceinline__ void epi_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kEpiThreads) : "memory"); }

// K-major operand tile with 64-byte swizzle (rows of 32 bf16): 8-row groups 512 B apart
__device__ __forceinline__ uint64_t sdesc_sw64(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(512 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)4 << 61;   // SWIZZLE_64B
  return d;
}

// ================================================================== GEMM
// 32 consecutive accumulator columns [n, n + 32) of row r (r < M) through the fused epilogue
// the chunk's bias, loaded before its accumulator columns are read from TMEM (the loads are in flight
// during the tcgen05.ld instead of stalling the epilogue after it)
__device__ __forceinline__ void bias_chunk(const SwGemm& g, int n, float4* b) {
#pragma unroll
  for (int c = 0; c < 8; ++c) b[c] = g.bias ? __ldg(reinterpret_cast<const float4*>(g.bias + n) + c) : make_float4(0.f, 0.f, 0.f, 0.f);
}

template <int EPI>
__device__ __forceinline__ void epi_chunk(const SwGemm& g, int r, int n, float* v, const float4* bq = nullptr) {
  if (bq) {
#pragma unroll
    for (int c = 0; c < 32; c += 4) {
      const float4 b = bq[c / 4];
      v[c] += b.x; v[c + 1] += b.y; v[c + 2] += b.z; v[c + 3] += b.w;
    }
  } else if (g.bias) {
    const float4* bp = reinterpret_cast<const float4*>(g.bias + n);
#pragma unroll
    for (int c = 0; c < 32; c += 4) {
      const float4 b = __ldg(bp + c / 4);
      v[c] += b.x; v[c + 1] += b.y; v[c + 2] += b.z; v[c + 3] += b.w;
    }
  }
  if constexpr (EPI == SWE_F32) {
    float4* dst = reinterpret_cast<float4*>(g.out_f + (int64_t)r * g.N + n);
#pragma unroll
    for (int c = 0; c < 32; c += 4) dst[c / 4] = make_float4(v[c], v[c + 1], v[c + 2], v[c + 3]);
  } else if constexpr (EPI == SWE_GELU) {
    uint4* dst = reinterpret_cast<uint4*>(g.out_b + (int64_t)r * g.N + n);
#pragma unroll
    for (int c = 0; c < 32; c += 8)
      dst[c / 8] = make_uint4(pack_gelu2(v[c], v[c + 1]), pack_gelu2(v[c + 2], v[c + 3]), pack_gelu2(v[c + 4], v[c + 5]),
                              pack_gelu2(v[c + 6], v[c + 7]));
  } else if constexpr (EPI == SWE_RESID) {
    const int tok = g.rowmap ? __ldg(g.rowmap + r) : r;
    float4* xp = reinterpret_cast<float4*>(g.out_f + (int64_t)tok * g.N + n);
    float4 x[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = xp[c];
#pragma unroll
    for (int c = 0; c < 8; ++c)
      xp[c] = make_float4(x[c].x + v[4 * c], x[c].y + v[4 * c + 1], x[c].z + v[4 * c + 2], x[c].w + v[4 * c + 3]);
  } else {   // SWE_QKV: the 32 columns are one head of q, k or v
    const int which = n / g.C, head = (n % g.C) >> 5;
    const int win = r / g.L2, i = r % g.L2;
    const int64_t unit = (int64_t)win * g.heads + head;
    if (which == 2) {
      uint16_t* dst = g.vt + unit * (32 * SW_WIN_ROWS) + i;
#pragma unroll
      for (int c = 0; c < 32; ++c) dst[c * SW_WIN_ROWS] = bf16_bits(v[c]);
    } else {
      const float s = which == 0 ? g.qscale : 1.f;
      uint4* dst = reinterpret_cast<uint4*>((which == 0 ? g.q : g.k) + (unit * SW_WIN_ROWS + i) * 32);
#pragma unroll
      for (int c = 0; c < 32; c += 8)
        dst[c / 8] = make_uint4(pack_bf16(v[c] * s, v[c + 1] * s), pack_bf16(v[c + 2] * s, v[c + 3] * s),
                                pack_bf16(v[c + 4] * s, v[c + 5] * s), pack_bf16(v[c + 6] * s, v[c + 7] * s));
    }
  }
}

// runtime dispatch (the 2-SM kernel serves every epilogue kind)
__device__ __forceinline__ void epi_chunk_rt(const SwGemm& g, int r, int n, float* v, const float4* bq = nullptr) {
  switch (g.epi) {
    case SWE_F32: epi_chunk<SWE_F32>(g, r, n, v, bq); break;
    case SWE_GELU: epi_chunk<SWE_GELU>(g, r, n, v, bq); break;
    case SWE_RESID: epi_chunk<SWE_RESID>(g, r, n, v, bq); break;
    default: epi_chunk<SWE_QKV>(g, r, n, v, bq); break;
  }
}

// ---- coalesced epilogue stores through a per-warp 2 KB staging tile (32 rows x 64 bytes).  A warp's
// accumulator chunk is one row per lane (32 rows x 32 columns); stored straight from registers every
// store instruction touches 32 rows (32 partial sectors).  Staged, lane l stores 16 bytes of row
// 8 j + l / 4 (j < 4): 8 rows x 64 contiguous bytes per instruction.  16-byte chunks are XOR-swizzled
// by row so both the row-per-lane writes and the row-major reads are bank-conflict free.
constexpr int kEpiStageBytes = 2048;
__device__ __forceinline__ void stg_put(char* stg, int lane, uint4 a, uint4 b, uint4 c, uint4 d) {
  const int sw = (lane >> 1) & 3;
  char* row = stg + lane * 64;
  *reinterpret_cast<uint4*>(row + ((0 ^ sw) << 4)) = a;
  *reinterpret_cast<uint4*>(row + ((1 ^ sw) << 4)) = b;
  *reinterpret_cast<uint4*>(row + ((2 ^ sw) << 4)) = c;
  *reinterpret_cast<uint4*>(row + ((3 ^ sw) << 4)) = d;
}
__device__ __forceinline__ uint4 stg_get(const char* stg, int row, int c) {
  return *reinterpret_cast<const uint4*>(stg + row * 64 + ((c ^ ((row >> 1) & 3)) << 4));
}
__device__ __forceinline__ uint4 f4u(float a, float b, float c, float d) {
  return make_uint4(__float_as_uint(a), __float_as_uint(b), __float_as_uint(c), __float_as_uint(d));
}

// one warp's 32 x 32 chunk (rows rbase + lane, columns [n, n + 32)), bias already added, through the
// staging tile.  RESID: tk[j] is the token row (window reverse + roll) of staged row 8 j + lane / 4 and
// x[h][j] its residual float4 at column group 16 h + 4 (lane % 4), loaded by the caller before the
// accumulator so the round trip overlaps the tcgen05.ld.
template <int EPI>
__device__ __forceinline__ void epi_staged(const SwGemm& g, int rbase, int lane, int n, const float* v, char* stg,
                                           const float4 (*x)[4], const int* tk) {
  const int cq = lane & 3;
  if constexpr (EPI == SWE_GELU || EPI == SWE_QKV) {
    // bf16 row of 32 columns = 64 bytes
    uint32_t u[16];
    const int which = EPI == SWE_QKV ? n / g.C : 0;
    const float sc = (EPI == SWE_QKV && which == 0) ? g.qscale : 1.f;
#pragma unroll
    for (int c = 0; c < 16; ++c)
      u[c] = EPI == SWE_GELU ? pack_gelu2(v[2 * c], v[2 * c + 1]) : pack_bf16(v[2 * c] * sc, v[2 * c + 1] * sc);
    __syncwarp();
    stg_put(stg, lane, make_uint4(u[0], u[1], u[2], u[3]), make_uint4(u[4], u[5], u[6], u[7]),
            make_uint4(u[8], u[9], u[10], u[11]), make_uint4(u[12], u[13], u[14], u[15]));
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int row = 8 * j + (lane >> 2), r = rbase + row;
      if (r >= g.M) continue;
      const uint4 val = stg_get(stg, row, cq);
      if constexpr (EPI == SWE_GELU) {
        *reinterpret_cast<uint4*>(g.out_b + (int64_t)r * g.N + n + 8 * cq) = val;
      } else {   // Q / K: head-major (window, head) unit rows of 32 bf16
        const int head = (n % g.C) >> 5, win = r / g.L2, i = r % g.L2;
        const int64_t unit = (int64_t)win * g.heads + head;
        *reinterpret_cast<uint4*>((which == 0 ? g.q : g.k) + (unit * SW_WIN_ROWS + i) * 32 + 8 * cq) = val;
      }
    }
  } else {
    // fp32 rows: two halves of 16 columns (64 bytes)
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const float* w = v + 16 * h;
      __syncwarp();
      stg_put(stg, lane, f4u(w[0], w[1], w[2], w[3]), f4u(w[4], w[5], w[6], w[7]), f4u(w[8], w[9], w[10], w[11]),
              f4u(w[12], w[13], w[14], w[15]));
      __syncwarp();
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int row = 8 * j + (lane >> 2), r = rbase + row;
        const uint4 val = stg_get(stg, row, cq);
        const float4 a = make_float4(__uint_as_float(val.x), __uint_as_float(val.y), __uint_as_float(val.z),
                                     __uint_as_float(val.w));
        if constexpr (EPI == SWE_RESID) {
          if (r < g.M) {
            const float4 xx = x[h][j];
            *reinterpret_cast<float4*>(g.out_f + (int64_t)tk[j] * g.N + n + 16 * h + 4 * cq) =
                make_float4(xx.x + a.x, xx.y + a.y, xx.z + a.z, xx.w + a.w);
          }
        } else {
          if (r < g.M) *reinterpret_cast<float4*>(g.out_f + (int64_t)r * g.N + n + 16 * h + 4 * cq) = a;
        }
      }
    }
  }
}

struct GemmCtrl {
  uint64_t full[8], empty[8], tfull[2], tempty[2];
  uint32_t tmem;
};

template <int EPI>   // the epilogue kind (g.epi): one specialised kernel per fused epilogue
__global__ void __launch_bounds__(SW_GEMM_THREADS, 1) sw_gemm_kernel(const __grid_constant__ GemmArgs A) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  GemmCtrl* C = reinterpret_cast<GemmCtrl*>(smem);
  char* ring = smem + 1024;
  const SwGemm& g = A.g;
  const int BN = g.BN, NS = g.stages, SP = g.splits;
  const uint32_t A_BYTES = 16384, STAGE = A_BYTES + (uint32_t)BN * 128;
  const int ntn = g.N / BN, tiles = ntn * ((g.M + 127) / 128), nk = g.K / 64 / SP;   // chunks per unit
  const int units = tiles * SP;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  pdl_trigger();
  if (threadIdx.x == 0) {
    for (int i = 0; i < NS; ++i) {
      ptx::mbar_init(&C->full[i], 1);
      ptx::mbar_init(&C->empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&C->tfull[i], 1);
      ptx::mbar_init(&C->tempty[i], kEpiThreads);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    ptx::prefetch_tmap(&A.ta);
    ptx::prefetch_tmap(&A.tb);
  }
  if (warp == 1) ptx::tmem_alloc(&C->tmem, (uint32_t)(2 * BN));
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = C->tmem;
  pdl_wait();   // the A operand / residual stream is written by the previous kernel
  trace_stamp(g.trace, g.op);

  if (warp == 0) {
    // ---- TMA producer: A [128 x 64] and W [BN x 64] K-chunks of every unit of this CTA
    uint32_t it = 0;
    for (int u = blockIdx.x; u < units; u += gridDim.x) {
      const int t = u / SP, kc0 = (u % SP) * nk;
      const int m0 = (t / ntn) * 128, n0 = (t % ntn) * BN;
      for (int kc = 0; kc < nk; ++kc, ++it) {
        const uint32_t slot = it % NS, ph = (it / NS) & 1;
        ptx::mbar_wait(&C->empty[slot], ph ^ 1);
        if (ptx::elect_one()) {
          char* st = ring + slot * STAGE;
          ptx::mbar_arrive_expect_tx(&C->full[slot], STAGE);
          ptx::tma_load_2d(st, &A.ta, &C->full[slot], (kc0 + kc) * 64, m0);
          ptx::tma_load_2d(st + A_BYTES, &A.tb, &C->full[slot], (kc0 + kc) * 64, n0);
        }
        __syncwarp();
      }
    }
  } else if (warp == 1) {
    // ---- MMA issuer: the whole warp runs the loop (uniform descriptors), one lane issues
    const uint32_t idesc = ptx::idesc_bf16(128, BN);
    const uint64_t d0 = ptx::sdesc_sw128(ptx::smem_u32(ring));
    uint32_t it = 0, lt = 0;
    for (int u = blockIdx.x; u < units; u += gridDim.x, ++lt) {
      const uint32_t buf = lt & 1, use = lt >> 1;
      ptx::mbar_wait(&C->tempty[buf], (use & 1) ^ 1);
      ptx::tc_fence_after();
      const uint32_t d = tmem + buf * BN;
      for (int kc = 0; kc < nk; ++kc, ++it) {
        const uint32_t slot = it % NS, ph = (it / NS) & 1;
        ptx::mbar_wait(&C->full[slot], ph);
        ptx::tc_fence_after();
        const uint64_t da = d0 + (uint64_t)((slot * STAGE) >> 4);
        const uint64_t db = da + (uint64_t)(A_BYTES >> 4);
        if (ptx::elect_one()) {
          ptx::mma_bf16_k64(d, da, db, idesc, kc > 0 ? 1u : 0u);
          ptx::mma_commit(&C->empty[slot]);
          if (kc == nk - 1) ptx::mma_commit(&C->tfull[buf]);
        }
        __syncwarp();
      }
    }
  } else {
    // ---- epilogue warps 2..: warp w reads TMEM lanes 32 * (w % 4) .. (its lane quarter); the
    // kEpiGroups warps of a quarter take interleaved 32-column chunks
    const int q = warp & 3, eh = (warp - 2) >> 2, et = threadIdx.x - 64;
    uint32_t lt = 0;
    for (int u = blockIdx.x; u < units; u += gridDim.x, ++lt) {
      const uint32_t buf = lt & 1, use = lt >> 1;
      const int t = u / SP, split = u % SP;
      const int m0 = (t / ntn) * 128, n0 = (t % ntn) * BN;
      ptx::mbar_wait(&C->tfull[buf], use & 1);
      ptx::tc_fence_after();
      const int rt = q * 32 + lane, r = m0 + rt;
      if (SP == 1 && !g.direct && EPI != SWE_QKV) {
        // staged (coalesced) stores (b64: FC1 -9 %, FC2 -13 %, proj -21 %); the QKV scatter keeps the
        // per-thread stores (each thread's 64-byte Q / K row segment is already whole sectors, and
        // staging measured +8 %)
        char* stg = ring + NS * STAGE + (warp - 2) * kEpiStageBytes;
        const int rbase = m0 + q * 32;
        int tk[4] = {0, 0, 0, 0};
        if (EPI == SWE_RESID)
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const int rr = rbase + 8 * j + (lane >> 2);
            tk[j] = rr < g.M ? (g.rowmap ? __ldg(g.rowmap + rr) : rr) : 0;
          }
        for (int c0 = 32 * eh; c0 < BN; c0 += 32 * kEpiGroups) {
          float v[32];
          float4 bq[8], x[2][4];
          bias_chunk(g, n0 + c0, bq);
          if (EPI == SWE_RESID)
#pragma unroll
            for (int h = 0; h < 2; ++h)
#pragma unroll
              for (int j = 0; j < 4; ++j)
                x[h][j] = rbase + 8 * j + (lane >> 2) < g.M
                              ? *reinterpret_cast<const float4*>(g.out_f + (int64_t)tk[j] * g.N + n0 + c0 + 16 * h + 4 * (lane & 3))
                              : make_float4(0.f, 0.f, 0.f, 0.f);
          ptx::tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + buf * BN + c0, v);
          if (EPI == SWE_QKV && (n0 + c0) / g.C == 2) {
            // V^T: for each column the warp's 32 rows are 64 contiguous bytes already
            if (r < g.M) epi_chunk<EPI>(g, r, n0 + c0, v, bq);
          } else {
#pragma unroll
            for (int c = 0; c < 8; ++c) {
              v[4 * c] += bq[c].x; v[4 * c + 1] += bq[c].y; v[4 * c + 2] += bq[c].z; v[4 * c + 3] += bq[c].w;
            }
            epi_staged<EPI>(g, rbase, lane, n0 + c0, v, stg, x, tk);
          }
        }
      } else if (SP == 1 && EPI == SWE_RESID) {
        // residual epilogue: the row's destination token (window reverse + roll) once per tile, and
        // each residual chunk loaded before its accumulator columns are read from TMEM, so the round
        // trip overlaps the tcgen05.ld (issued after it, it stalled every chunk)
        const int tok = r < g.M ? (g.rowmap ? __ldg(g.rowmap + r) : r) : 0;
        for (int c0 = 32 * eh; c0 < BN; c0 += 32 * kEpiGroups) {
          float v[32];
          float4 bq[8], x[8];
          bias_chunk(g, n0 + c0, bq);
          float4* xp = reinterpret_cast<float4*>(g.out_f + (int64_t)tok * g.N + n0 + c0);
          if (r < g.M) {
#pragma unroll
            for (int c = 0; c < 8; ++c) x[c] = xp[c];
          }
          ptx::tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + buf * BN + c0, v);
          if (r < g.M) {
#pragma unroll
            for (int c = 0; c < 8; ++c)
              xp[c] = make_float4(x[c].x + (v[4 * c] + bq[c].x), x[c].y + (v[4 * c + 1] + bq[c].y),
                                  x[c].z + (v[4 * c + 2] + bq[c].z), x[c].w + (v[4 * c + 3] + bq[c].w));
          }
        }
      } else
      for (int c0 = 32 * eh; c0 < BN; c0 += 32 * kEpiGroups) {
        float v[32];
        float4 bq[8];
        if (SP == 1) bias_chunk(g, n0 + c0, bq);
        ptx::tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + buf * BN + c0, v);
        if (SP == 1) {
          if (r < g.M) epi_chunk<EPI>(g, r, n0 + c0, v, bq);
        } else if (EPI == SWE_RESID) {
          // residual epilogue is linear: every split adds its partial (split 0 also the bias)
          // straight into the fp32 residual stream with vector atomics -- no partial round trip
          // (the order of the fp32 adds varies from run to run: ulp-level nondeterminism)
          if (r < g.M) {
            if (split == 0 && g.bias) {
              const float4* bp = reinterpret_cast<const float4*>(g.bias + n0 + c0);
#pragma unroll
              for (int c = 0; c < 32; c += 4) {
                const float4 b = __ldg(bp + c / 4);
                v[c] += b.x; v[c + 1] += b.y; v[c + 2] += b.z; v[c + 3] += b.w;
              }
            }
            const int tok = g.rowmap ? __ldg(g.rowmap + r) : r;
            float* xp = g.out_f + (int64_t)tok * g.N + n0 + c0;
#pragma unroll
            for (int c = 0; c < 32; c += 4)
              asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(xp + c), "f"(v[c]), "f"(v[c + 1]),
                           "f"(v[c + 2]), "f"(v[c + 3])
                           : "memory");
          }
        } else {   // fp32 partial of this split
          float4* dst = reinterpret_cast<float4*>(g.part + ((int64_t)u * 128 + rt) * BN + c0);
#pragma unroll
          for (int c = 0; c < 32; c += 4) dst[c / 4] = make_float4(v[c], v[c + 1], v[c + 2], v[c + 3]);
        }
      }
      ptx::tc_fence_before();
      ptx::mbar_arrive(&C->tempty[buf]);
      if (SP > 1 && EPI != SWE_RESID) {
        // meet the other splits of this tile (all units are co-resident: grid == units <= #SMs);
        // the barrier orders every epilogue thread's partial stores before thread et == 0's release
        epi_sync();
        if (et == 0) {
          ptx::red_release_add(&g.cnt[t], 1u);
          while (ptx::ld_acquire(&g.cnt[t]) < (unsigned)SP) {
          }
        }
        epi_sync();
        // reduce rows [split * 128 / SP, ...) of the tile, splits summed in order
        const int rows = 128 / SP, cpr = BN / 32;
        for (int item = et; item < rows * cpr; item += kEpiThreads) {
          const int rr = split * rows + item / cpr, c0 = (item % cpr) * 32;
          float v[32];
#pragma unroll
          for (int c = 0; c < 32; ++c) v[c] = 0.f;
          for (int k = 0; k < SP; ++k) {
            const float4* src = reinterpret_cast<const float4*>(g.part + ((int64_t)(t * SP + k) * 128 + rr) * BN + c0);
#pragma unroll
            for (int c = 0; c < 32; c += 4) {
              const float4 x = __ldcg(src + c / 4);
              v[c] += x.x; v[c + 1] += x.y; v[c + 2] += x.z; v[c + 3] += x.w;
            }
          }
          if (m0 + rr < g.M) epi_chunk<EPI>(g, m0 + rr, n0 + c0, v);
        }
        epi_sync();
        if (et == 0) {   // the last split to finish resets the tile's counters for the next run
          if (atomicAdd(&g.cnt[tiles + t], 1u) == (unsigned)SP - 1) {
            g.cnt[t] = 0u;
            g.cnt[tiles + t] = 0u;
          }
        }
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 1) ptx::tmem_dealloc(tmem, (uint32_t)(2 * BN));
}

// ================================================================== 2-SM GEMM (cta_group::2)
// For large M (batch >= 8): a CTA pair (cluster of 2, one TPC) computes a 256 x 256 tile with
// tcgen05.mma.cta_group::2 -- each CTA loads its 128 rows of A and HALF of the 256 W rows, the tensor
// cores of the pair read both halves, so every SM ingests 32 KB per 64-deep K chunk instead of 48 KB
// for the same MMA work (the 1-SM 128 x 256 tile is bound by per-SM operand ingest).  Both CTAs'
// TMA loads complete on the leader's barrier (.cta_group::2); rank 0 issues the MMAs; MMA completion
// is multicast to both CTAs' barriers; each CTA's epilogue drains its own 128 TMEM lanes.
struct Gemm2Ctrl {
  uint64_t full[8], empty[8], tfull[2], tempty[2];
  uint32_t tmem;
};
// TMA load into this CTA's shared memory whose completion is counted on an mbarrier of either CTA of
// the pair (`bar`: shared::cluster address)
__device__ __forceinline__ void tma2_load_2d(void* dst, const void* tmap, uint32_t bar, int32_t c0, int32_t c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          ptx::smem_u32(dst)),
      "l"(tmap), "r"(bar), "r"(c0), "r"(c1)
      : "memory");
}

__device__ __forceinline__ void mma2_bf16_k64(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                              uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .b64 a1, a2, a3, b1, b2, b3;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "setp.eq.b32 q, 0, 0;\n\t"
      "add.s64 a1, %1, 2;\n\tadd.s64 a2, %1, 4;\n\tadd.s64 a3, %1, 6;\n\t"
      "add.s64 b1, %2, 2;\n\tadd.s64 b2, %2, 4;\n\tadd.s64 b3, %2, 6;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], a1, b1, %3, q;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], a2, b2, %3, q;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], a3, b3, %3, q;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// MMA completion -> the same mbarrier offset in both CTAs of the pair
__device__ __forceinline__ void mma2_commit_both(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                   ptx::smem_u32(bar)),
               "h"((uint16_t)3)
               : "memory");
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
  asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}

__global__ void __launch_bounds__(SW_GEMM_THREADS, 1) sw_gemm2_kernel(const __grid_constant__ GemmArgs A) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  Gemm2Ctrl* C = reinterpret_cast<Gemm2Ctrl*>(smem);
  char* ring = smem + 1024;
  const SwGemm& g = A.g;
  constexpr int BN = 256;                     // pair tile: 256 rows x 256 columns
  constexpr uint32_t A_BYTES = 16384, B_BYTES = 16384, STAGE = A_BYTES + B_BYTES;
  const int NS = g.stages;
  const uint32_t rank = ptx::cluster_ctarank();
  const int pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;
  const int ntn = g.N / BN, tiles = ntn * ((g.M + 255) / 256), nk = g.K / 64;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  pdl_trigger();
  if (threadIdx.x == 0) {
    for (int i = 0; i < NS; ++i) {
      ptx::mbar_init(&C->full[i], 1);
      ptx::mbar_init(&C->empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      ptx::mbar_init(&C->tfull[i], 1);
      ptx::mbar_init(&C->tempty[i], 2 * kEpiThreads);   // both CTAs' epilogue threads (leader's copy)
    }
    ptx::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    ptx::prefetch_tmap(&A.ta);
    ptx::prefetch_tmap(&A.tb);
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(ptx::smem_u32(&C->tmem)),
                 "r"(2u * BN)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  ptx::tc_fence_before();
  __syncthreads();
  cluster_sync_all();   // both CTAs' barriers initialised before any remote arrive / multicast commit
  ptx::tc_fence_after();
  const uint32_t tmem = C->tmem;
  pdl_wait();
  trace_stamp(g.trace, g.op);
  const uint32_t leader_tempty[2] = {ptx::mapa(ptx::smem_u32(&C->tempty[0]), 0u), ptx::mapa(ptx::smem_u32(&C->tempty[1]), 0u)};

  if (warp == 0) {
    // ---- TMA producer: this CTA's 128 rows of A and its half (128 rows) of the 256 W rows; both
    // CTAs' loads complete on the LEADER's full barrier (.cta_group::2), which expects both halves
    const uint32_t full0 = ptx::mapa(ptx::smem_u32(&C->full[0]), 0u);
    uint32_t it = 0;
    for (int t = pair; t < tiles; t += npairs) {
      const int m0 = (t / ntn) * 256 + (int)rank * 128, n0 = (t % ntn) * BN + (int)rank * 128;
      for (int kc = 0; kc < nk; ++kc, ++it) {
        const uint32_t slot = it % NS, ph = (it / NS) & 1;
        ptx::mbar_wait(&C->empty[slot], ph ^ 1);
        if (ptx::elect_one()) {
          char* st = ring + slot * STAGE;
          const uint32_t bar = full0 + slot * 8;
          if (rank == 0) ptx::mbar_arrive_expect_tx(&C->full[slot], 2 * STAGE);
          tma2_load_2d(st, &A.ta, bar, kc * 64, m0);
          tma2_load_2d(st + A_BYTES, &A.tb, bar, kc * 64, n0);
        }
        __syncwarp();
      }
    }
  } else if (warp == 1) {
    uint32_t it = 0, lt = 0;
    if (rank == 0) {
      // ---- leader: MMA issue (M = 256 across the pair, N = 256, K = 16)
      const uint32_t idesc = ptx::idesc_bf16(256, BN);
      const uint64_t d0 = ptx::sdesc_sw128(ptx::smem_u32(ring));
      for (int t = pair; t < tiles; t += npairs, ++lt) {
        const uint32_t buf = lt & 1, use = lt >> 1;
        ptx::mbar_wait_cluster(&C->tempty[buf], (use & 1) ^ 1);
        ptx::tc_fence_after();
        const uint32_t d = tmem + buf * BN;
        for (int kc = 0; kc < nk; ++kc, ++it) {
          const uint32_t slot = it % NS, ph = (it / NS) & 1;
          ptx::mbar_wait(&C->full[slot], ph);
          ptx::tc_fence_after();
          const uint64_t da = d0 + (uint64_t)((slot * STAGE) >> 4);
          const uint64_t db = da + (uint64_t)(A_BYTES >> 4);
          if (ptx::elect_one()) {
            mma2_bf16_k64(d, da, db, idesc, kc > 0 ? 1u : 0u);
            mma2_commit_both(&C->empty[slot]);
            if (kc == nk - 1) mma2_commit_both(&C->tfull[buf]);
          }
          __syncwarp();
        }
      }
    }
  } else {
    // ---- epilogue: this CTA's 128 rows of the pair tile (its own TMEM lanes)
    const int q = warp & 3, eh = (warp - 2) >> 2;
    uint32_t lt = 0;
    for (int t = pair; t < tiles; t += npairs, ++lt) {
      const uint32_t buf = lt & 1, use = lt >> 1;
      const int m0 = (t / ntn) * 256 + (int)rank * 128, n0 = (t % ntn) * BN;
      ptx::mbar_wait(&C->tfull[buf], use & 1);
      ptx::tc_fence_after();
      const int r = m0 + q * 32 + lane;
      for (int c0 = 32 * eh; c0 < BN; c0 += 32 * kEpiGroups) {
        float v[32];
        float4 bq[8];
        bias_chunk(g, n0 + c0, bq);
        ptx::tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + buf * BN + c0, v);
        if (r < g.M) epi_chunk_rt(g, r, n0 + c0, v, bq);
      }
      ptx::tc_fence_before();
      ptx::mbar_arrive_remote(leader_tempty[buf]);   // the leader's MMA reuses this buffer
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  cluster_sync_all();   // the peer's TMEM / smem are not released while the pair still uses them
  if (warp == 1)
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(2u * BN) : "memory");
}

// ================================================================== window attention
struct AttnCtrl {
  uint64_t ld[2], mma, tb;
  uint32_t tmem;
};
constexpr int kAttnTile = 8192;   // Q pair, K pair, V^T pair: 8 KB each
constexpr int kTabBytes = 2 * SW_TAB * 4;   // the pair's two score-bias tiles

__global__ void __launch_bounds__(SW_ATTN_THREADS) sw_attn_kernel(const __grid_constant__ AttnArgs A) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  AttnCtrl* C = reinterpret_cast<AttnCtrl*>(smem);
  char* Ps = smem + 1024;                      // [128 rows][128 keys] bf16: 2 SW128 atoms of 16 KB
  char* tiles = Ps + 32768;                    // 2 buffers x (Q, K, V^T)
  float* tab = reinterpret_cast<float*>(tiles + 2 * 3 * kAttnTile);   // the pair's score-bias tiles
  const SwAttn& a = A.a;
  const int pairs = a.units / 2;
  const int tid = threadIdx.x, warp = tid >> 5;
  pdl_trigger();
  if (tid == 0) {
    ptx::mbar_init(&C->ld[0], 1);
    ptx::mbar_init(&C->ld[1], 1);
    ptx::mbar_init(&C->mma, 1);
    ptx::mbar_init(&C->tb, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 0) ptx::tmem_alloc(&C->tmem, 256);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = C->tmem;   // S: columns [0, 128); O: [128, 160)
  pdl_wait();
  trace_stamp(a.trace, a.op);
  auto issue = [&](int p, int b) {
    char* t = tiles + b * 3 * kAttnTile;
    ptx::mbar_arrive_expect_tx(&C->ld[b], 3 * kAttnTile);
    ptx::tma_load_2d(t, &A.tq, &C->ld[b], 0, p * 128);
    ptx::tma_load_2d(t + kAttnTile, &A.tk, &C->ld[b], 0, p * 128);
    ptx::tma_load_2d(t + 2 * kAttnTile, &A.tv, &C->ld[b], 0, p * 64);
  };
  // the pair's two (window, head) tiles of the score-bias table: units 2p, 2p+1 are heads h, h+1 of
  // one window, contiguous in tab[window % nW][heads]
  auto issue_tab = [&](int p) {
    const int unit = 2 * p, win = unit / a.heads, head = unit % a.heads;
    const float* src = a.tab + ((int64_t)(win % a.nW) * a.heads + head) * SW_TAB;
    ptx::mbar_arrive_expect_tx(&C->tb, kTabBytes);
    ptx::bulk_g2s(tab, src, kTabBytes, &C->tb);
  };
  if (tid == 0 && (int)blockIdx.x < pairs) {
    issue(blockIdx.x, 0);
    issue_tab(blockIdx.x);
  }
  const int r = tid, uh = r >> 6, i = r & 63;   // row of the tile: unit half, token in the window
  uint32_t it = 0, mph = 0;
  const float L2E = 1.4426950408889634f;
  for (int p = blockIdx.x; p < pairs; p += gridDim.x, ++it) {
    const int b = it & 1;
    char* t = tiles + b * 3 * kAttnTile;
    if (tid == 0 && p + (int)gridDim.x < pairs) issue(p + gridDim.x, b ^ 1);   // next pair's tiles
    ptx::mbar_wait(&C->ld[b], (it >> 1) & 1);
    // ---- S = Q K^T: M = 128 (two units), N = 128 keys, K = 32 (two K = 16 steps of 32 bytes)
    if (warp == 0) {
      ptx::tc_fence_after();
      const uint64_t dq = sdesc_sw64(ptx::smem_u32(t)), dk = sdesc_sw64(ptx::smem_u32(t + kAttnTile));
      if (ptx::elect_one()) {
        ptx::mma_bf16(tmem, dq, dk, ptx::idesc_bf16(128, 128), 0u);
        ptx::mma_bf16(tmem, dq + 2, dk + 2, ptx::idesc_bf16(128, 128), 1u);
        ptx::mma_commit(&C->mma);
      }
      __syncwarp();
    }
    const int unit = 2 * p + uh, win = unit / a.heads, head = unit % a.heads;
    const float* trow = tab + uh * SW_TAB + i * a.L2;   // this row's additive terms (smem)
    ptx::mbar_wait(&C->tb, it & 1);
    ptx::mbar_wait(&C->mma, mph);
    mph ^= 1;
    ptx::tc_fence_after();
    float s[64];
    ptx::tmem_ld64(tmem + ((uint32_t)(warp * 32) << 16) + uh * 64, s);
    const bool live = i < a.L2;
    float mx = -INFINITY;
#pragma unroll
    for (int j = 0; j < 64; ++j) {
      if (live && j < a.L2) {
        s[j] = (s[j] + trow[j]) * L2E;
      } else {
        s[j] = -INFINITY;
      }
      mx = fmaxf(mx, s[j]);
    }
    float z = 0.f;
    if (live) {
#pragma unroll
      for (int j = 0; j < 64; ++j) {
        s[j] = ptx::ex2(s[j] - mx);
        z += s[j];
      }
    }
    const float iz = live ? 1.f / z : 0.f;
    // P row r: this unit's 64 keys in atom uh, zeros in the other atom (block-diagonal pair)
#pragma unroll
    for (int c0 = 0; c0 < 64; c0 += 8) {
      *reinterpret_cast<uint4*>(Ps + uh * 16384 + sw128(r, c0 * 2)) =
          live ? make_uint4(pack_bf16(s[c0] * iz, s[c0 + 1] * iz), pack_bf16(s[c0 + 2] * iz, s[c0 + 3] * iz),
                            pack_bf16(s[c0 + 4] * iz, s[c0 + 5] * iz), pack_bf16(s[c0 + 6] * iz, s[c0 + 7] * iz))
               : make_uint4(0u, 0u, 0u, 0u);
      *reinterpret_cast<uint4*>(Ps + (uh ^ 1) * 16384 + sw128(r, c0 * 2)) = make_uint4(0u, 0u, 0u, 0u);
    }
    ptx::tc_fence_before();
    ptx::fence_proxy_async_smem();
    __syncthreads();
    // the table is consumed: fetch the next pair's (it lands during PV and the stores)
    if (tid == 0 && p + (int)gridDim.x < pairs) issue_tab(p + gridDim.x);
    // ---- O = P V: M = 128, N = 32, K = 128 keys (atom 0 = unit A's keys with its V^T, atom 1 = B's)
    if (warp == 0) {
      ptx::tc_fence_after();
      const uint64_t dp = ptx::sdesc_sw128(ptx::smem_u32(Ps)), dv = ptx::sdesc_sw128(ptx::smem_u32(t + 2 * kAttnTile));
      if (ptx::elect_one()) {
        ptx::mma_bf16_k64(tmem + 128, dp, dv, ptx::idesc_bf16(128, 32), 0u);
        ptx::mma_bf16_k64(tmem + 128, dp + (16384 >> 4), dv + (4096 >> 4), ptx::idesc_bf16(128, 32), 1u);
        ptx::mma_commit(&C->mma);
      }
      __syncwarp();
    }
    ptx::mbar_wait(&C->mma, mph);
    mph ^= 1;
    ptx::tc_fence_after();
    float o[32];
    ptx::tmem_ld32(tmem + 128 + ((uint32_t)(warp * 32) << 16), o);
    ptx::tc_fence_before();
    if (live) {
      uint4* dst = reinterpret_cast<uint4*>(a.ctx + ((int64_t)win * a.L2 + i) * a.C + head * 32);
#pragma unroll
      for (int c = 0; c < 32; c += 8)
        dst[c / 8] = make_uint4(pack_bf16(o[c], o[c + 1]), pack_bf16(o[c + 2], o[c + 3]), pack_bf16(o[c + 4], o[c + 5]),
                                pack_bf16(o[c + 6], o[c + 7]));
    }
    __syncthreads();   // S / O / P reused by the next pair
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) ptx::tmem_dealloc(tmem, 256);
}

// ================================================================== LayerNorm of gathered rows
// One warp per output row; lane l holds float4 column groups l, l + 32, ... (NV groups).  The
// statistics are merged pairwise (Chan) from exactly centred per-lane values: a constant row gives
// exactly beta, an offset row keeps its noise (no E[x^2] - E[x]^2 cancellation).
// RPW rows per warp (narrow rows: C = 128 or 256): every row's gather-index loads are issued, then every
// row's data loads, so a warp keeps RPW x NV float4 requests in flight instead of NV (the narrow stages
// were bound by the bytes in flight per SM, not by HBM).
template <int NV, int RPW>
__global__ void __launch_bounds__(SW_ROW_THREADS) sw_row_kernel(const SwRow R) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  pdl_trigger();
  pdl_wait();
  trace_stamp(R.trace, R.op);
  const int rbase = (blockIdx.x * (SW_ROW_THREADS / 32) + warp) * RPW;
  if (rbase >= R.rows) return;
  const int cin = R.cols / R.nsrc;
  int tok[RPW][NV];
#pragma unroll
  for (int q = 0; q < RPW; ++q)
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      const int r = min(rbase + q, R.rows - 1);
      const int e = 4 * (lane + 32 * k);
      const int s = e / cin;
      tok[q][k] = R.src ? __ldg(R.src + (int64_t)r * R.nsrc + s) : r;
    }
  float4 v[RPW][NV];
#pragma unroll
  for (int q = 0; q < RPW; ++q)
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      const int e = 4 * (lane + 32 * k);
      const int s = e / cin, o = e - s * cin;
      v[q][k] = __ldg(reinterpret_cast<const float4*>(R.x + (int64_t)tok[q][k] * cin + o));
    }
#pragma unroll
  for (int q = 0; q < RPW; ++q) {
    const int r = rbase + q;
    float m = 0.f;
#pragma unroll
    for (int k = 0; k < NV; ++k) m += (v[q][k].x + v[q][k].y) + (v[q][k].z + v[q][k].w);
    m *= 1.f / (float)(4 * NV);
    float M2 = 0.f;
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      const float a = v[q][k].x - m, b = v[q][k].y - m, c = v[q][k].z - m, d = v[q][k].w - m;
      M2 += (a * a + b * b) + (c * c + d * d);
    }
    float n = (float)(4 * NV);
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const float mb = __shfl_xor_sync(0xffffffffu, m, o), Mb = __shfl_xor_sync(0xffffffffu, M2, o);
      const float dl = mb - m;
      M2 = (M2 + Mb) + dl * dl * (0.5f * n);
      m = (m + mb) * 0.5f;
      n *= 2.f;
    }
    if (r >= R.rows) continue;
    const float rs = rsqrtf(M2 / (float)R.cols + R.eps);
#pragma unroll
    for (int k = 0; k < NV; ++k) {
      const int e = 4 * (lane + 32 * k);
      const float4 gm = __ldg(reinterpret_cast<const float4*>(R.gamma + e));
      const float4 bt = __ldg(reinterpret_cast<const float4*>(R.beta + e));
      const float4 y = make_float4((v[q][k].x - m) * rs * gm.x + bt.x, (v[q][k].y - m) * rs * gm.y + bt.y,
                                   (v[q][k].z - m) * rs * gm.z + bt.z, (v[q][k].w - m) * rs * gm.w + bt.w);
      if (R.out_b)
        *reinterpret_cast<uint2*>(R.out_b + (int64_t)r * R.cols + e) = make_uint2(pack_bf16(y.x, y.y), pack_bf16(y.z, y.w));
      if (R.out_f) *reinterpret_cast<float4*>(R.out_f + (int64_t)r * R.cols + e) = y;
    }
  }
}

// ================================================================== score-bias tables
__global__ void sw_bias_kernel(const SwBias B) {
  pdl_trigger();
  pdl_wait();
  trace_stamp(B.trace, B.op);
  const SwBiasEnt& E = B.ent[blockIdx.y];
  const int L2 = B.L2, L22 = L2 * L2;
  constexpr int G = SW_TAB / 4;   // float4 groups per (window, head) tile
  const int64_t n = (int64_t)E.nW * E.heads * G;
  for (int64_t o = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; o < n; o += (int64_t)gridDim.x * blockDim.x) {
    const int g = (int)(o % G);
    const int64_t u = o / G;           // (w, h) unit of the table
    const int h = (int)(u % E.heads), w = (int)(u / E.heads);
    float v[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int t = 4 * g + e;
      v[e] = 0.f;
      if (t < L22) {
        v[e] = __ldg(E.bias + (int64_t)h * L22 + t);
        if (E.mask) v[e] += __ldg(E.mask + (int64_t)w * L22 + t);
      }
    }
    reinterpret_cast<float4*>(E.dst)[o] = make_float4(v[0], v[1], v[2], v[3]);
  }
}

// ================================================================== patch embedding gather
// thread per (token, 4-column group): groups 0..11 = (c, kh) rows of the 4 x 4 patch (one float4 of
// the image row), 12..15 = zero padding of K to 64
__global__ void sw_im2col_kernel(const SwIm2col P) {
  pdl_trigger();
  pdl_wait();
  trace_stamp(P.trace, P.op);
  const int64_t T = (int64_t)P.B * P.R * P.R;
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx < (int64_t)P.C * 64) {   // padded weight copy [C][64]
    const int row = (int)(idx / 64), col = (int)(idx % 64);
    P.wpad[idx] = col < 48 ? P.w[row * 48 + col] : (uint16_t)0;
  }
  if (idx >= T * 16) return;
  const int g = (int)(idx % 16);
  const int64_t tok = idx / 16;
  float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
  if (g < 12) {
    const int b = (int)(tok / (P.R * P.R)), ty = (int)(tok / P.R % P.R), tx = (int)(tok % P.R);
    const int c = g >> 2, kh = g & 3;
    v = __ldg(reinterpret_cast<const float4*>(P.image + (((int64_t)b * 3 + c) * P.img + ty * 4 + kh) * P.img + tx * 4));
  }
  reinterpret_cast<uint2*>(P.out)[idx] = make_uint2(pack_bf16(v.x, v.y), pack_bf16(v.z, v.w));
}

// ================================================================== final LN + mean pool + head
__global__ void __launch_bounds__(256) sw_pool_kernel(const SwHead H) {
  extern __shared__ float hsm[];          // [8][C] per-warp pooled sums
  pdl_trigger();
  pdl_wait();
  trace_stamp(H.trace, H.op);
  const int b = blockIdx.x, warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int C = H.C, NV = C / 128;
  for (int c = threadIdx.x; c < 8 * C; c += 256) hsm[c] = 0.f;
  __syncthreads();
  for (int t = warp; t < H.L; t += 8) {
    const float* xr = H.x + ((int64_t)b * H.L + t) * C;
    float4 v[8];
    float m = 0.f;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      v[k] = k < NV ? __ldg(reinterpret_cast<const float4*>(xr) + lane + 32 * k) : make_float4(0.f, 0.f, 0.f, 0.f);
      m += (v[k].x + v[k].y) + (v[k].z + v[k].w);
    }
    m *= 1.f / (float)(4 * NV);
    float M2 = 0.f, n = (float)(4 * NV);
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      if (k < NV) {
        const float a = v[k].x - m, bb = v[k].y - m, c = v[k].z - m, d = v[k].w - m;
        M2 += (a * a + bb * bb) + (c * c + d * d);
      }
    }
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const float mb = __shfl_xor_sync(0xffffffffu, m, o), Mb = __shfl_xor_sync(0xffffffffu, M2, o);
      const float dl = mb - m;
      M2 = (M2 + Mb) + dl * dl * (0.5f * n);
      m = (m + mb) * 0.5f;
      n *= 2.f;
    }
    const float rs = rsqrtf(M2 / (float)C + H.eps);
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      if (k >= NV) break;
      const int e = 4 * (lane + 32 * k);
      const float4 gm = __ldg(reinterpret_cast<const float4*>(H.gamma + e));
      const float4 bt = __ldg(reinterpret_cast<const float4*>(H.beta + e));
      float* p = hsm + warp * C + e;
      p[0] += (v[k].x - m) * rs * gm.x + bt.x;
      p[1] += (v[k].y - m) * rs * gm.y + bt.y;
      p[2] += (v[k].z - m) * rs * gm.z + bt.z;
      p[3] += (v[k].w - m) * rs * gm.w + bt.w;
    }
  }
  __syncthreads();
  for (int c = threadIdx.x; c < C; c += 256) {
    float s = 0.f;
#pragma unroll
    for (int w = 0; w < 8; ++w) s += hsm[w * C + c];
    H.pooled[(int64_t)b * C + c] = bf2f(bf16_bits(s / (float)H.L));   // bf16 matmul operand
  }
}

// a warp per class: the class's weight row stays in registers, dotted with every image's pooled row
__global__ void __launch_bounds__(256) sw_head_kernel(const SwHead H) {
  pdl_trigger();
  pdl_wait();
  trace_stamp(H.trace, H.op);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n = blockIdx.x * 8 + warp;
  if (n >= H.classes) return;
  const int C = H.C;
  float w[32];   // C <= 1024: 32 weights per lane, columns lane * 8 + 256 * j + e
  const uint16_t* wr = H.W + (int64_t)n * C;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    uint4 w8 = make_uint4(0u, 0u, 0u, 0u);
    if (lane * 8 + 256 * j < C) w8 = __ldg(reinterpret_cast<const uint4*>(wr + lane * 8 + 256 * j));
    const uint32_t ws[4] = {w8.x, w8.y, w8.z, w8.w};
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      w[8 * j + 2 * e] = __uint_as_float(ws[e] << 16);
      w[8 * j + 2 * e + 1] = __uint_as_float(ws[e] & 0xffff0000u);
    }
  }
  const float bias = __ldg(H.bias + n);
  for (int b0 = 0; b0 < H.B; b0 += 4) {   // 4 images at a time: independent loads in flight
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int bb = 0; bb < 4; ++bb) {
      if (b0 + bb >= H.B) break;
      const float* pr = H.pooled + (int64_t)(b0 + bb) * C;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (lane * 8 + 256 * j < C) {
          const float4 p0 = __ldcg(reinterpret_cast<const float4*>(pr + lane * 8 + 256 * j));
          const float4 p1 = __ldcg(reinterpret_cast<const float4*>(pr + lane * 8 + 256 * j + 4));
          acc[bb] += p0.x * w[8 * j] + p0.y * w[8 * j + 1] + p0.z * w[8 * j + 2] + p0.w * w[8 * j + 3] +
                     p1.x * w[8 * j + 4] + p1.y * w[8 * j + 5] + p1.z * w[8 * j + 6] + p1.w * w[8 * j + 7];
        }
      }
    }
#pragma unroll
    for (int bb = 0; bb < 4; ++bb) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) acc[bb] += __shfl_xor_sync(0xffffffffu, acc[bb], o);
      if (lane == 0 && b0 + bb < H.B) H.out[(int64_t)(b0 + bb) * H.classes + n] = acc[bb] + bias;
    }
  }
}

}  // namespace swin

// ------------------------------------------------------------------ host-side launchers
// every launch allows programmatic dependent launch: the next kernel's CTAs start (prologue: barrier
// init, TMEM alloc, tensor-map prefetch) while this one drains, and wait in griddepcontrol.wait
template <typename... KArgs, typename... Args>
static cudaError_t launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k, std::forward<Args>(args)...);
}

// dynamic shared-memory opt-in, once per kernel (the largest configuration any launch uses)
static cudaError_t set_smem(const void* f, int bytes) {
  static const void* done[8] = {};
  for (const void* d : done)
    if (d == f) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess)
    for (auto& d : done)
      if (!d) { d = f; break; }
  return e;
}

int sw_gemm_smem(int BN, int stages) { return 2048 + stages * (16384 + BN * 128); }
int sw_gemm1_smem(int BN, int stages) { return sw_gemm_smem(BN, stages) + swin::kEpiWarps * swin::kEpiStageBytes; }
int sw_attn_smem() { return 2048 + 32768 + 2 * 3 * swin::kAttnTile + swin::kTabBytes; }

cudaError_t sw_launch_gemm(const void* ta, const void* tb, const SwGemm& g, int grid, cudaStream_t s) {
  swin::GemmArgs a;
  memcpy(&a.ta, ta, sizeof(CUtensorMap));
  memcpy(&a.tb, tb, sizeof(CUtensorMap));
  a.g = g;
  void (*fn)(swin::GemmArgs) = g.epi == SWE_F32    ? swin::sw_gemm_kernel<SWE_F32>
                               : g.epi == SWE_GELU ? swin::sw_gemm_kernel<SWE_GELU>
                               : g.epi == SWE_RESID ? swin::sw_gemm_kernel<SWE_RESID>
                                                    : swin::sw_gemm_kernel<SWE_QKV>;
  cudaError_t e = set_smem((const void*)fn, 227 * 1024);
  if (e != cudaSuccess) return e;
  return launch_pdl(fn, dim3(grid), dim3(SW_GEMM_THREADS), (size_t)sw_gemm1_smem(g.BN, g.stages), s, a);
}

cudaError_t sw_launch_gemm2(const void* ta, const void* tb, const SwGemm& g, int grid, cudaStream_t s) {
  swin::GemmArgs a;
  memcpy(&a.ta, ta, sizeof(CUtensorMap));
  memcpy(&a.tb, tb, sizeof(CUtensorMap));
  a.g = g;
  cudaError_t e = set_smem((const void*)swin::sw_gemm2_kernel, 227 * 1024);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(SW_GEMM_THREADS);
  cfg.dynamicSmemBytes = (size_t)sw_gemm_smem(128, g.stages);   // 32 KB stages
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  at[1].id = cudaLaunchAttributeClusterDimension;
  at[1].val.clusterDim.x = 2;
  at[1].val.clusterDim.y = 1;
  at[1].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, swin::sw_gemm2_kernel, a);
}

cudaError_t sw_launch_attn(const void* tq, const void* tk, const void* tv, const SwAttn& at, int grid, cudaStream_t s) {
  swin::AttnArgs a;
  memcpy(&a.tq, tq, sizeof(CUtensorMap));
  memcpy(&a.tk, tk, sizeof(CUtensorMap));
  memcpy(&a.tv, tv, sizeof(CUtensorMap));
  a.a = at;
  const int sm = sw_attn_smem();
  cudaError_t e = set_smem((const void*)swin::sw_attn_kernel, sm);
  if (e != cudaSuccess) return e;
  return launch_pdl(swin::sw_attn_kernel, dim3(grid), dim3(SW_ATTN_THREADS), (size_t)sm, s, a);
}

cudaError_t sw_launch_row(const SwRow& r, cudaStream_t s) {
  // rows per warp: 4 for C = 128, 2 for C = 256 (SOUFFLE_SWIN_LN_RPW1=1: one row per warp, studies)
  static const bool one = std::getenv("SOUFFLE_SWIN_LN_RPW1") != nullptr;
  int rpw = one ? 1 : r.cols == 128 ? 4 : r.cols == 256 ? 2 : 1;
  if ((r.rows + 8 * rpw - 1) / (8 * rpw) < 2 * 148) rpw = 1;   // small batches: keep the CTAs (b1: -1 %)
  const dim3 grid((r.rows + 8 * rpw - 1) / (8 * rpw)), blk(SW_ROW_THREADS);
  switch (r.cols / 128) {
    case 1: return rpw == 4 ? launch_pdl(swin::sw_row_kernel<1, 4>, grid, blk, 0, s, r)
                            : launch_pdl(swin::sw_row_kernel<1, 1>, grid, blk, 0, s, r);
    case 2: return rpw == 2 ? launch_pdl(swin::sw_row_kernel<2, 2>, grid, blk, 0, s, r)
                            : launch_pdl(swin::sw_row_kernel<2, 1>, grid, blk, 0, s, r);
    case 4: return launch_pdl(swin::sw_row_kernel<4, 1>, grid, blk, 0, s, r);
    case 8: return launch_pdl(swin::sw_row_kernel<8, 1>, grid, blk, 0, s, r);
    case 16: return launch_pdl(swin::sw_row_kernel<16, 1>, grid, blk, 0, s, r);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t sw_launch_bias(const SwBias& b, int max_table, cudaStream_t s) {
  return launch_pdl(swin::sw_bias_kernel, dim3((unsigned)std::max(1, std::min(256, max_table / 4 / 256)), b.n), dim3(256), 0,
                    s, b);
}

cudaError_t sw_launch_im2col(const SwIm2col& p, cudaStream_t s) {
  const int64_t n = std::max<int64_t>((int64_t)p.B * p.R * p.R * 16, (int64_t)p.C * 64);
  return launch_pdl(swin::sw_im2col_kernel, dim3((unsigned)((n + 255) / 256)), dim3(256), 0, s, p);
}

cudaError_t sw_launch_pool(const SwHead& h, cudaStream_t s) {
  cudaError_t e = set_smem((const void*)swin::sw_pool_kernel, 8 * 1024 * 4);
  if (e != cudaSuccess) return e;
  return launch_pdl(swin::sw_pool_kernel, dim3(h.B), dim3(256), (size_t)(8 * h.C * 4), s, h);
}

cudaError_t sw_launch_head(const SwHead& h, cudaStream_t s) {
  return launch_pdl(swin::sw_head_kernel, dim3((h.classes + 7) / 8), dim3(256), 0, s, h);
}

}  // namespace souffle
