// The Souffle subprogram executor for sm_100a (B200).
//
// One persistent cooperative kernel runs a whole subprogram (§4, §6.4
// P:L1169-1176): it walks the subprogram's stage list, each CTA takes tasks of the current stage,
// and a grid barrier separates stages with a dependence ("global sync", Fig. 2).  Stage
// kinds:
//   ST_GEMM_TC   tcgen05 bf16 GEMM (M=128 tiles, TMEM accumulator, TMA + mbarrier ring), split-K
//                partials combined with fp32 atomics and finished by the last-arriving CTA,
//                fused epilogue program (vertical transformation) and fused row reductions
//                (two-phase reduction, §2.3 P:L527-536 / §6.3)
//   ST_ATTN      QK^T -> softmax -> PV per head on tcgen05, S and O in TMEM, P in smem (Fig. 1(c))
//   ST_GEMM_SIMT fp32 FFMA GEMM with the same epilogue programs (fp32 graphs, GEMVs, batched)
//   ST_EW        vertically fused one-relies-on-one chain (§6.2) over a 2-D domain
//   ST_REDUCE    one reduction with fused producer / consumer chains
// The fused chains are executed by a small vector interpreter over CHUNK columns (the index maps
// of §5.2 are pre-enumerated on the host into affine / separable / full offset tables).
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../exec_types.h"
#include "ptx.cuh"

namespace souffle {

constexpr int kThreads = EXEC_THREADS;
constexpr int kSlots = 4;              // TC ring slots (A 16 KB + B 16 KB each)
constexpr int kSlotBytes = 32768;
constexpr int kCtrlBytes = 1024;       // mbarriers + TMEM address at the start of smem

struct SmemCtrl {
  uint64_t full[kSlots];
  uint64_t empty[kSlots];
  uint64_t accb;
  uint64_t attb;
  uint32_t tmem_base;
  int32_t flag;
};

struct TcState {
  uint32_t it_p, it_c;       // producer / consumer iteration counters of the smem ring
  uint32_t acc_phase;        // parity of the accumulator barrier
  uint32_t att_phase;
};

// ================================================================== element access
__device__ __forceinline__ int64_t addr_off(const Params& P, const Addr& A, int64_t r, int64_t c) {
  if (A.mode == 0) return A.base + r * A.rs + c * A.cs;
  if (A.mode == 1) return A.base + P.tabs[A.rtab + r] + P.tabs[A.ctab + c];
  return A.base + P.tabs[A.ftab + r * A.ncols + c];
}
__device__ __forceinline__ char* addr_ptr(const Params& P, const Addr& A) {
  return A.buf >= 0 ? (char*)P.bufs[A.buf] : P.ws_data;
}
__device__ __forceinline__ float bf2f(uint16_t b) { return __uint_as_float(((uint32_t)b) << 16); }
__device__ __forceinline__ uint16_t f2bf(float f) {
  __nv_bfloat16 h = __float2bfloat16_rn(f);
  return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float ld_elem(const Params& P, const Addr& A, int64_t r, int64_t c) {
  int64_t o = addr_off(P, A, r, c);
  char* p = addr_ptr(P, A);
  if (A.dtype == 0) {
    const float* f = (const float*)p + o;
    return A.cg ? __ldcg(f) : __ldg(f);
  }
  const unsigned short* h = (const unsigned short*)p + o;
  return bf2f(A.cg ? __ldcg(h) : __ldg(h));
}
__device__ __forceinline__ void st_elem(const Params& P, const Addr& A, int64_t r, int64_t c, float v) {
  int64_t o = addr_off(P, A, r, c);
  char* p = addr_ptr(P, A);
  if (A.dtype == 0) ((float*)p)[o] = v;
  else ((uint16_t*)p)[o] = f2bf(v);
}

// ================================================================== chain interpreter
__device__ __forceinline__ float fn_un(int fn, float x) {
  switch (fn) {
    case FN_EXP: return expf(x);
    case FN_TANH: return tanhf(x);
    case FN_SIGMOID: return 1.f / (1.f + expf(-x));
    case FN_RELU: return x > 0.f ? x : 0.f;
    case FN_GELU: return 0.5f * x * (1.f + erff(x * 0.70710678118654752f));
    case FN_RSQRT: return rsqrtf(x);
    case FN_NEG: return -x;
  }
  return x;
}
__device__ __forceinline__ float fn_bin(int fn, float a, float b) {
  switch (fn) {
    case FN_ADD: return a + b;
    case FN_SUB: return a - b;
    case FN_MUL: return a * b;
    case FN_DIV: return a / b;
    case FN_MAX: return fmaxf(a, b);
  }
  return a;
}

template <int W>
struct Regs {
  float v[NREG][W];
};

template <int W, class F>
__device__ __forceinline__ void with_reg(Regs<W>& R, int a, F f) {
  switch (a) {
    case 0: f(R.v[0]); break;
    case 1: f(R.v[1]); break;
    case 2: f(R.v[2]); break;
    default: f(R.v[3]); break;
  }
}

// Runs a fused-chain program at domain row r, columns c0 .. c0+nvalid-1.  acc[] = accumulator
// values of those columns.  Row reductions accumulate into red[] (caller flushes).
template <int W>
__device__ void run_prog(const Params& P, int prog, int len, int64_t r, int64_t c0, int nvalid, const float* acc,
                         float* red) {
  Regs<W> R;
#pragma unroll
  for (int k = 0; k < NREG; ++k)
#pragma unroll
    for (int j = 0; j < W; ++j) R.v[k][j] = 0.f;
  for (int i = 0; i < len; ++i) {
    const Ins I = P.ins[prog + i];
    switch (I.op) {
      case OP_LOAD: {
        const Addr& A = P.addrs[I.addr];
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] = j < nvalid ? ld_elem(P, A, r, c0 + j) : 0.f;
        });
        break;
      }
      case OP_ACC:
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] = acc[j];
        });
        break;
      case OP_UN:
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] = fn_un(I.fn, x[j]);
        });
        break;
      case OP_SCAL:
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] = I.fn == FN_ADDS ? x[j] + I.imm : x[j] * I.imm;
        });
        break;
      case OP_BIN:
      case OP_BINR: {
        float t[W];
        with_reg<W>(R, I.b, [&](float* y) {
#pragma unroll
          for (int j = 0; j < W; ++j) t[j] = y[j];
        });
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] = I.op == OP_BINR ? fn_bin(I.fn, t[j], x[j]) : fn_bin(I.fn, x[j], t[j]);
        });
        break;
      }
      case OP_MOV: {
        float t[W];
        with_reg<W>(R, I.b, [&](float* y) {
#pragma unroll
          for (int j = 0; j < W; ++j) t[j] = y[j];
        });
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] = t[j];
        });
        break;
      }
      case OP_BINL: {
        const Addr& A = P.addrs[I.addr];
        float t[W];
#pragma unroll
        for (int j = 0; j < W; ++j) t[j] = j < nvalid ? ld_elem(P, A, r, c0 + j) : 0.f;
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] = I.b ? fn_bin(I.fn, t[j], x[j]) : fn_bin(I.fn, x[j], t[j]);
        });
        break;
      }
      case OP_STORE: {
        const Addr& A = P.addrs[I.addr];
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j)
            if (j < nvalid) st_elem(P, A, r, c0 + j, x[j]);
        });
        break;
      }
      case OP_RED: {
        float s = 0.f;
        with_reg<W>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < W; ++j)
            if (j < nvalid) s += x[j];
        });
        red[I.b] += s * I.imm;
        break;
      }
    }
  }
}

// flush per-thread partial row reductions (one atomic per row and reduction, §6.3)
__device__ void flush_reds(const Params& P, int prog, int len, int64_t r, float* red) {
  for (int i = 0; i < len; ++i) {
    const Ins I = P.ins[prog + i];
    if (I.op != OP_RED) continue;
    const Addr& A = P.addrs[I.addr];
    float* p = (float*)addr_ptr(P, A) + addr_off(P, A, r, 0);
    atomicAdd(p, red[I.b]);
    red[I.b] = 0.f;
  }
}

// ================================================================== grid barrier
__device__ __forceinline__ void grid_barrier(const Params& P, unsigned& nb) {
  __syncthreads();
  ++nb;
  if (threadIdx.x == 0) {
    __threadfence();
    ptx::fence_proxy_async();
    ptx::red_release_add(&P.ctrl[0], 1u);
    const unsigned target = nb * gridDim.x;
    while (ptx::ld_acquire(&P.ctrl[0]) < target) {
    }
    __threadfence();
  }
  __syncthreads();
  ptx::fence_proxy_async();
}

// ================================================================== EW stage
__device__ void run_ew(const Params& P, const Stage& st) {
  const int64_t cpr = (st.cols + CHUNK - 1) / CHUNK;
  const int64_t total = (int64_t)st.rows * cpr;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  for (int64_t t = (int64_t)blockIdx.x * kThreads + threadIdx.x; t < total; t += (int64_t)gridDim.x * kThreads) {
    int64_t r = t / cpr;
    int64_t c0 = (t % cpr) * CHUNK;
    int nv = (int)((st.cols - c0) < CHUNK ? (st.cols - c0) : CHUNK);
    float acc[CHUNK] = {0, 0, 0, 0, 0, 0, 0, 0};
    run_prog<CHUNK>(P, st.prog, st.prog_len, r, c0, nv, acc, red);
    flush_reds(P, st.prog, st.prog_len, r, red);
  }
}

// evaluate a program and return register 0 (used by reduction pre-programs)
__device__ void eval_r0(const Params& P, int prog, int len, int64_t r, int64_t c0, int nvalid, float* out) {
  Regs<CHUNK> R;
#pragma unroll
  for (int k = 0; k < NREG; ++k)
#pragma unroll
    for (int j = 0; j < CHUNK; ++j) R.v[k][j] = 0.f;
  for (int i = 0; i < len; ++i) {
    const Ins I = P.ins[prog + i];
    switch (I.op) {
      case OP_LOAD: {
        const Addr& A = P.addrs[I.addr];
        with_reg<CHUNK>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < CHUNK; ++j) x[j] = j < nvalid ? ld_elem(P, A, r, c0 + j) : 0.f;
        });
        break;
      }
      case OP_UN:
        with_reg<CHUNK>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < CHUNK; ++j) x[j] = fn_un(I.fn, x[j]);
        });
        break;
      case OP_SCAL:
        with_reg<CHUNK>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < CHUNK; ++j) x[j] = I.fn == FN_ADDS ? x[j] + I.imm : x[j] * I.imm;
        });
        break;
      case OP_BIN:
      case OP_BINR: {
        float t[CHUNK];
        with_reg<CHUNK>(R, I.b, [&](float* y) {
#pragma unroll
          for (int j = 0; j < CHUNK; ++j) t[j] = y[j];
        });
        with_reg<CHUNK>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < CHUNK; ++j) x[j] = I.op == OP_BINR ? fn_bin(I.fn, t[j], x[j]) : fn_bin(I.fn, x[j], t[j]);
        });
        break;
      }
      case OP_MOV: {
        float t[CHUNK];
        with_reg<CHUNK>(R, I.b, [&](float* y) {
#pragma unroll
          for (int j = 0; j < CHUNK; ++j) t[j] = y[j];
        });
        with_reg<CHUNK>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < CHUNK; ++j) x[j] = t[j];
        });
        break;
      }
      case OP_BINL: {
        const Addr& A = P.addrs[I.addr];
        float t[CHUNK];
#pragma unroll
        for (int j = 0; j < CHUNK; ++j) t[j] = j < nvalid ? ld_elem(P, A, r, c0 + j) : 0.f;
        with_reg<CHUNK>(R, I.a, [&](float* x) {
#pragma unroll
          for (int j = 0; j < CHUNK; ++j) x[j] = I.b ? fn_bin(I.fn, t[j], x[j]) : fn_bin(I.fn, x[j], t[j]);
        });
        break;
      }
      default: break;
    }
  }
#pragma unroll
  for (int j = 0; j < CHUNK; ++j) out[j] = R.v[0][j];
}

// ================================================================== REDUCE stage (warp per row)
__device__ void run_reduce(const Params& P, const Stage& st) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  for (int64_t o = (int64_t)blockIdx.x * 8 + warp; o < st.rows; o += (int64_t)gridDim.x * 8) {
    float acc = st.red_fn ? -INFINITY : 0.f;
    for (int64_t c0 = (int64_t)lane * CHUNK; c0 < st.cols; c0 += 32 * CHUNK) {
      int nv = (int)((st.cols - c0) < CHUNK ? (st.cols - c0) : CHUNK);
      float vals[CHUNK];
      eval_r0(P, st.prog, st.prog_len, o, c0, nv, vals);
#pragma unroll
      for (int j = 0; j < CHUNK; ++j)
        if (j < nv) acc = st.red_fn ? fmaxf(acc, vals[j]) : acc + vals[j];
    }
#pragma unroll
    for (int s = 16; s > 0; s >>= 1) {
      float y = __shfl_xor_sync(0xffffffffu, acc, s);
      acc = st.red_fn ? fmaxf(acc, y) : acc + y;
    }
    acc *= st.red_scale;
    if (lane == 0) {
      float a1[1] = {acc};
      run_prog<1>(P, st.post, st.post_len, o, 0, 1, a1, red);
      flush_reds(P, st.post, st.post_len, o, red);
    }
  }
}

// ================================================================== SIMT GEMM stage
__device__ void run_gemm_simt(const Params& P, const Stage& st, char* smem) {
  float(*As)[68] = reinterpret_cast<float(*)[68]>(smem);
  float(*Bs)[68] = reinterpret_cast<float(*)[68]>(smem + 16 * 68 * 4);
  const int tid = threadIdx.x, ty = tid >> 3, tx = tid & 7;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  for (int task = blockIdx.x; task < st.ntasks; task += gridDim.x) {
    int mi = 0;
    while (mi + 1 < st.nmem && P.members[st.mem0 + mi + 1].task0 <= task) ++mi;
    const GemmMember& G = P.members[st.mem0 + mi];
    const int local = task - G.task0;
    const int tmi = local / G.tiles_n, tn = local % G.tiles_n;
    const int mt = (G.M + 63) / 64;
    const int b = tmi / mt, tm = tmi % mt;
    const Addr& A = P.addrs[G.a_addr];
    const Addr& B = P.addrs[G.b_addr];
    float acc[2][8];
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
    for (int k0 = 0; k0 < G.K; k0 += 16) {
      __syncthreads();
      for (int e = tid; e < 16 * 64; e += kThreads) {
        int kk = e >> 6, i = e & 63;
        int m = tm * 64 + i, n = tn * 64 + i, k = k0 + kk;
        float av = 0.f, bv = 0.f;
        if (m < G.M && k < G.K) av = ld_elem(P, A, (int64_t)b * G.M + m, k);
        if (n < G.N && k < G.K) bv = ld_elem(P, B, (int64_t)b * G.N + n, k);
        if (G.prec) {
          av = __bfloat162float(__float2bfloat16_rn(av));
          bv = __bfloat162float(__float2bfloat16_rn(bv));
        }
        As[kk][i] = av;
        Bs[kk][i] = bv;
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < 16; ++kk) {
        float a0 = As[kk][ty * 2], a1 = As[kk][ty * 2 + 1];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          float bv = Bs[kk][tx * 8 + j];
          acc[0][j] = fmaf(a0, bv, acc[0][j]);
          acc[1][j] = fmaf(a1, bv, acc[1][j]);
        }
      }
    }
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      int m = tm * 64 + ty * 2 + i;
      int c0 = tn * 64 + tx * 8;
      if (m < G.M && c0 < G.N) {
        int nv = min(8, G.N - c0);
        int64_t r = (int64_t)b * G.M + m;
        run_prog<CHUNK>(P, G.prog, G.prog_len, r, c0, nv, acc[i], red);
        flush_reds(P, G.prog, G.prog_len, r, red);
      }
    }
  }
  __syncthreads();
}

// ================================================================== TC GEMM stage
// swizzled (128B) byte offset of element (row, k) inside a K-major tile with 64-element rows
__device__ __forceinline__ uint32_t sw128(int row, int kbyte) {
  return (uint32_t)(row * 128 + ((((kbyte >> 4) ^ (row & 7)) & 7) << 4) + (kbyte & 15));
}

__device__ void run_gemm_tc(const Params& P, const Stage& st, char* smem, SmemCtrl* ctl, TcState& ts) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  char* ring = smem + kCtrlBytes;
  const char* tmaps = (const char*)P.tmaps;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  for (int task = blockIdx.x; task < st.ntasks; task += gridDim.x) {
    int mi = 0;
    while (mi + 1 < st.nmem && P.members[st.mem0 + mi + 1].task0 <= task) ++mi;
    const GemmMember& G = P.members[st.mem0 + mi];
    const int local = task - G.task0;
    const int split = local % G.splits;
    const int tile = local / G.splits;
    const int tm = tile / G.tiles_n, tn = tile % G.tiles_n;
    const int NT = G.n_tile;
    const int rows = G.M * G.batch;
    const int m0 = tm * 128, n0 = tn * NT;
    const int kbeg = split * G.k_split;
    const int kend = min(G.K, kbeg + G.k_split);
    const int nk = (kend - kbeg) / 64;
    const uint32_t a_bytes = 128 * 128, b_bytes = (uint32_t)NT * 128;
    const bool tma_a = G.a_tmap >= 0;

    if (warp == 0) {
      // ---------------- producer: TMA (and manual fp32->bf16 A staging) into the ring
      for (int i = 0; i < nk; ++i) {
        const uint32_t slot = ts.it_p % kSlots, ph = (ts.it_p / kSlots) & 1;
        char* sa = ring + slot * kSlotBytes;
        char* sb = sa + 16384;
        if (lane == 0) ptx::mbar_wait(&ctl->empty[slot], ph ^ 1);
        __syncwarp();
        if (!tma_a) {
          const Addr& A = P.addrs[G.a_f32];
          for (int e = lane; e < 128 * 16; e += 32) {   // 128 rows x 16 groups of 4 floats
            int row = e >> 4, g4 = e & 15;
            int m = m0 + row, k = kbeg + i * 64 + g4 * 4;
            float v0 = 0.f, v1 = 0.f, v2 = 0.f, v3 = 0.f;
            if (m < rows) {
              v0 = ld_elem(P, A, m, k);
              v1 = ld_elem(P, A, m, k + 1);
              v2 = ld_elem(P, A, m, k + 2);
              v3 = ld_elem(P, A, m, k + 3);
            }
            uint32_t lo = (uint32_t)f2bf(v0) | ((uint32_t)f2bf(v1) << 16);
            uint32_t hi = (uint32_t)f2bf(v2) | ((uint32_t)f2bf(v3) << 16);
            *reinterpret_cast<uint2*>(sa + sw128(row, g4 * 8)) = make_uint2(lo, hi);
          }
          ptx::fence_proxy_async();
          __syncwarp();
        }
        if (lane == 0) {
          ptx::mbar_arrive_expect_tx(&ctl->full[slot], (tma_a ? a_bytes : 0) + b_bytes);
          if (tma_a) ptx::tma_load_2d(sa, tmaps + 128 * G.a_tmap, &ctl->full[slot], kbeg + i * 64, m0);
          ptx::tma_load_2d(sb, tmaps + 128 * G.b_tmap, &ctl->full[slot], kbeg + i * 64, n0);
        }
        __syncwarp();
        ++ts.it_p;
      }
    } else if (warp == 1) {
      // ---------------- MMA issuer (one thread)
      const uint32_t idesc = ptx::idesc_bf16(128, NT);
      for (int i = 0; i < nk; ++i) {
        const uint32_t slot = ts.it_c % kSlots, ph = (ts.it_c / kSlots) & 1;
        if (lane == 0) {
          ptx::mbar_wait(&ctl->full[slot], ph);
          ptx::tc_fence_after();
          const uint32_t sa = ptx::smem_u32(ring + slot * kSlotBytes);
          const uint32_t sb = sa + 16384;
#pragma unroll
          for (int k = 0; k < 4; ++k)
            ptx::mma_bf16(ctl->tmem_base, ptx::sdesc_sw128(sa + k * 32), ptx::sdesc_sw128(sb + k * 32), idesc,
                          (i > 0 || k > 0) ? 1u : 0u);
          ptx::mma_commit(&ctl->empty[slot]);
          if (i == nk - 1) ptx::mma_commit(&ctl->accb);
        }
        __syncwarp();
        ++ts.it_c;
      }
    } else if (warp >= 4) {
      // ---------------- epilogue warps: TMEM -> registers -> program / split-K partials
      const int q = warp - 4;
      const int row = q * 32 + lane;
      const int64_t r = m0 + row;
      ptx::mbar_wait(&ctl->accb, ts.acc_phase);
      ptx::tc_fence_after();
      const uint32_t tbase = ctl->tmem_base + ((uint32_t)(q * 32) << 16);
      if (G.splits == 1) {
        for (int c0 = 0; c0 < NT; c0 += 8) {
          float v[8];
          ptx::tmem_ld8(tbase + c0, v);
          if (r < rows) run_prog<CHUNK>(P, G.prog, G.prog_len, r, n0 + c0, 8, v, red);
        }
        if (r < rows) flush_reds(P, G.prog, G.prog_len, r, red);
      } else {
        float* accbuf = (float*)P.ws_data + G.acc_off + (int64_t)tile * 128 * NT + (int64_t)row * NT;
        for (int c0 = 0; c0 < NT; c0 += 8) {
          float v[8];
          ptx::tmem_ld8(tbase + c0, v);
          if (r < rows) {
            atomicAdd(reinterpret_cast<float4*>(accbuf + c0), make_float4(v[0], v[1], v[2], v[3]));
            atomicAdd(reinterpret_cast<float4*>(accbuf + c0 + 4), make_float4(v[4], v[5], v[6], v[7]));
          }
        }
        __threadfence();
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (threadIdx.x == 128) {
          unsigned* cnt = (unsigned*)P.ws_data + G.cnt_off + tile;
          unsigned old = atomicAdd(cnt, 1u);
          ctl->flag = (old == (unsigned)(G.splits - 1)) ? 1 : 0;
          if (ctl->flag) *cnt = 0u;   // self-cleaning for the next run
        }
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (ctl->flag) {
          __threadfence();
          if (r < rows) {
            for (int c0 = 0; c0 < NT; c0 += 8) {
              float4 x0 = __ldcg(reinterpret_cast<const float4*>(accbuf + c0));
              float4 x1 = __ldcg(reinterpret_cast<const float4*>(accbuf + c0 + 4));
              float v[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
              __stcg(reinterpret_cast<float4*>(accbuf + c0), make_float4(0.f, 0.f, 0.f, 0.f));
              __stcg(reinterpret_cast<float4*>(accbuf + c0 + 4), make_float4(0.f, 0.f, 0.f, 0.f));
              run_prog<CHUNK>(P, G.prog, G.prog_len, r, n0 + c0, 8, v, red);
            }
            flush_reds(P, G.prog, G.prog_len, r, red);
          }
        }
      }
      ptx::tc_fence_before();
    }
    ts.acc_phase ^= 1;
    __syncthreads();
  }
}

// ================================================================== ATTN stage
__device__ void run_attn(const Params& P, const Stage& st, char* smem, SmemCtrl* ctl, TcState& ts) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, tid = threadIdx.x;
  char* base = smem + kCtrlBytes;
  char* Qs = base;               // [128 q][d] K-major, d/64 atoms of 16 KB
  char* Ks = base + 32768;       // [128 keys][d]
  char* Vt = base + 65536;       // [d][128 keys], 2 atoms of d*128 B
  char* Ps = base + 98304;       // [128 q][128 keys], 2 atoms of 16 KB
  const int S = st.at_S, d = st.at_d;
  const int datoms = d / 64;
  const Addr& AQ = P.addrs[st.at_q];
  const Addr& AK = P.addrs[st.at_k];
  const Addr& AV = P.addrs[st.at_v];
  const uint16_t* gq = (const uint16_t*)addr_ptr(P, AQ) + AQ.base;
  const uint16_t* gk = (const uint16_t*)addr_ptr(P, AK) + AK.base;
  const uint16_t* gv = (const uint16_t*)addr_ptr(P, AV) + AV.base;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  const float scale = st.at_scale;
  for (int b = blockIdx.x; b < st.at_B; b += gridDim.x) {
    const int64_t hb = (int64_t)b * S * d;
    // ---- stage Q, K (K-major, swizzled) and V^T
    const int chunks = 128 * (d / 8);
    for (int e = tid; e < chunks; e += kThreads) {
      int s = e / (d / 8), c8 = e % (d / 8);
      int atom = c8 / 8, cb = (c8 % 8) * 16;
      uint4 qv = make_uint4(0, 0, 0, 0), kv = make_uint4(0, 0, 0, 0), vv = make_uint4(0, 0, 0, 0);
      if (s < S) {
        qv = __ldcg(reinterpret_cast<const uint4*>(gq + hb + (int64_t)s * d + c8 * 8));
        kv = __ldcg(reinterpret_cast<const uint4*>(gk + hb + (int64_t)s * d + c8 * 8));
        vv = __ldcg(reinterpret_cast<const uint4*>(gv + hb + (int64_t)s * d + c8 * 8));
      }
      *reinterpret_cast<uint4*>(Qs + atom * 16384 + sw128(s, cb)) = qv;
      *reinterpret_cast<uint4*>(Ks + atom * 16384 + sw128(s, cb)) = kv;
      // V^T: element (key s, dim c8*8+j) -> row (dim), column key
      const uint16_t* vp = reinterpret_cast<const uint16_t*>(&vv);
      int katom = s / 64, kb = (s % 64) * 2;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        int dd = c8 * 8 + j;
        *reinterpret_cast<uint16_t*>(Vt + katom * (d * 128) + sw128(dd, kb)) = vp[j];
      }
    }
    ptx::fence_proxy_async();
    __syncthreads();
    // ---- S = Q K^T  (M=128 queries, N=128 keys, K=d) -> TMEM cols [0,128)
    if (warp == 1 && lane == 0) {
      ptx::tc_fence_after();
      const uint32_t idesc = ptx::idesc_bf16(128, 128);
      const uint32_t q0 = ptx::smem_u32(Qs), k0 = ptx::smem_u32(Ks);
      for (int ks = 0; ks < d / 16; ++ks) {
        uint32_t off = (ks / 4) * 16384 + (ks % 4) * 32;
        ptx::mma_bf16(ctl->tmem_base, ptx::sdesc_sw128(q0 + off), ptx::sdesc_sw128(k0 + off), idesc, ks > 0);
      }
      ptx::mma_commit(&ctl->attb);
    }
    __syncwarp();
    // ---- softmax in registers (one thread per query row), P -> smem as bf16
    if (warp < 4) {
      ptx::mbar_wait(&ctl->attb, ts.att_phase);
      ptx::tc_fence_after();
      const int row = warp * 32 + lane;
      const uint32_t tb = ctl->tmem_base + ((uint32_t)(warp * 32) << 16);
      float mx = -INFINITY;
      for (int c0 = 0; c0 < 128; c0 += 8) {
        float v[8];
        ptx::tmem_ld8(tb + c0, v);
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if (c0 + j < S) mx = fmaxf(mx, v[j] * scale);
      }
      float z = 0.f;
      for (int c0 = 0; c0 < 128; c0 += 8) {
        float v[8];
        ptx::tmem_ld8(tb + c0, v);
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if (c0 + j < S) z += expf(v[j] * scale - mx);
      }
      const float iz = 1.f / z;
      for (int c0 = 0; c0 < 128; c0 += 8) {
        float v[8];
        ptx::tmem_ld8(tb + c0, v);
        uint32_t pk[4];
#pragma unroll
        for (int j = 0; j < 8; j += 2) {
          float p0 = (c0 + j < S) ? expf(v[j] * scale - mx) * iz : 0.f;
          float p1 = (c0 + j + 1 < S) ? expf(v[j + 1] * scale - mx) * iz : 0.f;
          pk[j / 2] = (uint32_t)f2bf(p0) | ((uint32_t)f2bf(p1) << 16);
        }
        int atom = c0 / 64, cb = (c0 % 64) * 2;
        *reinterpret_cast<uint4*>(Ps + atom * 16384 + sw128(row, cb)) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      }
      ptx::tc_fence_before();
    }
    ts.att_phase ^= 1;
    ptx::fence_proxy_async();
    __syncthreads();
    // ---- O = P V  (M=128, N=d, K=128 keys) -> TMEM cols [128, 128+d)
    if (warp == 1 && lane == 0) {
      ptx::tc_fence_after();
      const uint32_t idesc = ptx::idesc_bf16(128, d);
      const uint32_t p0 = ptx::smem_u32(Ps), v0 = ptx::smem_u32(Vt);
      for (int ks = 0; ks < 8; ++ks) {
        uint32_t pa = (ks / 4) * 16384 + (ks % 4) * 32;
        uint32_t va = (ks / 4) * (d * 128) + (ks % 4) * 32;
        ptx::mma_bf16(ctl->tmem_base + 128, ptx::sdesc_sw128(p0 + pa), ptx::sdesc_sw128(v0 + va), idesc, ks > 0);
      }
      ptx::mma_commit(&ctl->attb);
    }
    __syncwarp();
    if (warp >= 4) {
      const int q = warp - 4;
      ptx::mbar_wait(&ctl->attb, ts.att_phase);
      ptx::tc_fence_after();
      const int row = q * 32 + lane;
      const uint32_t tb = ctl->tmem_base + 128 + ((uint32_t)(q * 32) << 16);
      for (int c0 = 0; c0 < d; c0 += 8) {
        float v[8];
        ptx::tmem_ld8(tb + c0, v);
        if (row < S) run_prog<CHUNK>(P, st.prog, st.prog_len, (int64_t)b * S + row, c0, 8, v, red);
      }
      if (row < S) flush_reds(P, st.prog, st.prog_len, (int64_t)b * S + row, red);
      ptx::tc_fence_before();
    }
    ts.att_phase ^= 1;
    __syncthreads();
    (void)datoms;
  }
}

// ================================================================== the persistent kernel
__global__ void __launch_bounds__(kThreads, 1) souffle_exec_kernel(const __grid_constant__ Params P) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  SmemCtrl* ctl = reinterpret_cast<SmemCtrl*>(smem);
  const int warp = threadIdx.x >> 5;
  TcState ts{0u, 0u, 0u, 0u};
  if (P.uses_tc) {
    if (threadIdx.x == 0) {
      for (int s = 0; s < kSlots; ++s) {
        ptx::mbar_init(&ctl->full[s], 1);
        ptx::mbar_init(&ctl->empty[s], 1);
      }
      ptx::mbar_init(&ctl->accb, 1);
      ptx::mbar_init(&ctl->attb, 1);
      ptx::fence_mbar_init();
    }
    if (warp == 0) ptx::tmem_alloc(&ctl->tmem_base, 256);
    ptx::tc_fence_before();
    __syncthreads();
    ptx::tc_fence_after();
  }
  unsigned nb = 0;
  for (int s = P.first; s < P.first + P.count; ++s) {
    const Stage& st = P.stages[s];
    if (st.barrier_before && P.cooperative) grid_barrier(P, nb);
    switch (st.kind) {
      case ST_EW: run_ew(P, st); break;
      case ST_REDUCE: run_reduce(P, st); break;
      case ST_GEMM_SIMT: run_gemm_simt(P, st, smem + kCtrlBytes); break;
      case ST_GEMM_TC: run_gemm_tc(P, st, smem, ctl, ts); break;
      case ST_ATTN: run_attn(P, st, smem, ctl, ts); break;
    }
  }
  // ---- exit: the last CTA resets the barrier words and clears the fused-reduction targets
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    unsigned old = atomicAdd(&P.ctrl[1], 1u);
    ctl->flag = (old == gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  if (ctl->flag) {
    __threadfence();
    if (P.is_last) {
      for (int z = 0; z < P.n_zero; ++z) {
        float4* p = reinterpret_cast<float4*>(P.ws_data + P.zero_list[2 * z]);
        int64_t n4 = P.zero_list[2 * z + 1] / 16;
        for (int64_t i = threadIdx.x; i < n4; i += kThreads) __stcg(p + i, make_float4(0.f, 0.f, 0.f, 0.f));
      }
    }
    if (threadIdx.x == 0) {
      P.ctrl[0] = 0u;
      P.ctrl[1] = 0u;
    }
  }
  if (P.uses_tc) {
    ptx::tc_fence_before();
    __syncthreads();
    if (warp == 0) ptx::tmem_dealloc(ctl->tmem_base, 256);
  }
}

cudaError_t exec_launch(const Params& prm, int grid, int smem, bool cooperative, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(souffle_exec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, EXEC_SMEM + 1024);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = EXEC_SMEM + 1024;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = cooperative ? 1 : 0;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  (void)smem;
  return cudaLaunchKernelEx(&cfg, souffle_exec_kernel, prm);
}

cudaError_t exec_max_active(int smem, int* blocks) {
  cudaError_t e = cudaFuncSetAttribute(souffle_exec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, EXEC_SMEM + 1024);
  if (e != cudaSuccess) return e;
  (void)smem;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, souffle_exec_kernel, kThreads, EXEC_SMEM + 1024);
}

}  // namespace souffle
