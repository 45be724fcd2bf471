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
// The fused chains are executed by a small vector interpreter over CHUNK columns.  Programs and
// their address records (index maps of §5.2 pre-enumerated on the host into affine / separable /
// full offset tables) are staged in shared memory per stage, and every chunk issues all of its
// global loads as one batch before computing (memory-level parallelism instead of a dependent
// load chain per instruction).
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../exec_types.h"
#include "ptx.cuh"

namespace souffle {

constexpr int kThreads = EXEC_THREADS;
constexpr int kSlots = 4;              // TC ring slots (A 16 KB + B 16 KB each)
constexpr int kSlotBytes = 32768;
constexpr int kCtrlBytes = 8192;       // control block + staged stage descriptor + program caches
constexpr int kCacheIns = 64;
constexpr int kCacheAddr = 32;
constexpr int kMaxPf = 6;              // batched loads per chunk

struct TcState {
  uint32_t it_p, it_c;       // producer / consumer iteration counters of the smem ring
  uint32_t acc_phase;        // parity of the accumulator barrier
  uint32_t att_phase;
};

struct SmemCtrl {
  uint64_t full[kSlots];
  uint64_t empty[kSlots];
  uint64_t accb;
  uint64_t attb;
  uint32_t tmem_base;
  int32_t flag;
  TcState ts;
  int32_t cur_stage;
  int32_t pf_member;     // GEMM member of this CTA's first task, prefetched with its program
  GemmMember mem;        // its record
};
static_assert(sizeof(SmemCtrl) <= 512, "SmemCtrl must fit below the staged stage descriptor");
static_assert(512 + sizeof(Stage) <= 1024, "stage descriptor must fit below the program caches");
static_assert(sizeof(Stage) % 16 == 0 && sizeof(Addr) % 8 == 0, "staged with vector copies");

// debug timeline mark k of the current stage (CTA 0 only; the calling thread decides who marks),
// plus a per-CTA copy of marks 0..3 at prof[9*nst + 1 + (stage*kProfCtas + cta)*4 + k]
constexpr int kProfCtas = 160;
__device__ __forceinline__ void mark(const Params& P, const SmemCtrl* ctl, int k) {
  if (P.prof) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (blockIdx.x == 0) P.prof[P.n_stages_total + 1 + 8 * ctl->cur_stage + k] = t;
    if (k <= 5 && blockIdx.x < kProfCtas)   // per CTA: marks 0,1,2 and the last of 3/4/5 (work done)
      P.prof[9 * P.n_stages_total + 1 + ((int64_t)ctl->cur_stage * kProfCtas + blockIdx.x) * 4 + (k < 3 ? k : 3)] = t;
  }
}

struct Prog {
  const Ins* ins;
  const Addr* addr;
  const FastPath* fast;
  int len;
};

struct ProgCache {
  Ins ins[kCacheIns];
  Addr addr[kCacheAddr];
  FastPath fast;
  Prog p;      // the staged program (points into this cache, or to global memory if too large)
};

__device__ __forceinline__ SmemCtrl* ctrl_of(char* smem) { return reinterpret_cast<SmemCtrl*>(smem); }
__device__ __forceinline__ Stage* stage_of(char* smem) { return reinterpret_cast<Stage*>(smem + 512); }
__device__ __forceinline__ ProgCache* cache_of(char* smem, int k) {
  return reinterpret_cast<ProgCache*>(smem + 1024 + k * (int)sizeof(ProgCache));
}
static_assert(1024 + 2 * sizeof(ProgCache) <= kCtrlBytes, "control block overflow");
static_assert(kCtrlBytes + kSlots * kSlotBytes <= EXEC_SMEM, "smem budget");

// Stage a program into a smem cache (all threads of the CTA must call; ends with __syncthreads).
__device__ Prog stage_prog(const Params& P, const ProgRef& R, ProgCache* c) {
  Prog p;
  p.len = R.len;
  if (R.len <= kCacheIns && R.naddr <= kCacheAddr) {
    const int4* si = reinterpret_cast<const int4*>(P.ins + R.ins0);
    int4* di = reinterpret_cast<int4*>(c->ins);
    const int nI = R.len * (int)sizeof(Ins) / 16;
    for (int i = threadIdx.x; i < nI; i += kThreads) di[i] = si[i];
    const int64_t* sa = reinterpret_cast<const int64_t*>(P.addrs + R.addr0);
    int64_t* da = reinterpret_cast<int64_t*>(c->addr);
    const int nA = R.naddr * (int)sizeof(Addr) / 8;
    for (int i = threadIdx.x; i < nA; i += kThreads) da[i] = sa[i];
    p.ins = c->ins;
    p.addr = c->addr;
  } else {
    p.ins = P.ins + R.ins0;
    p.addr = P.addrs + R.addr0;
  }
  p.fast = &c->fast;
  if (threadIdx.x == 0) {
    c->fast = R.fast;
    c->p = p;
  }
  __syncthreads();
  return p;
}

// ================================================================== element access
__device__ __forceinline__ int64_t addr_off(const Params& P, const Addr& A, int64_t r, int64_t c) {
  if (A.mode == 0) return A.base + r * A.rs + c * A.cs;
  if (A.mode == 1) return A.base + P.tabs[A.rtab + r] + P.tabs[A.ctab + c];
  return A.base + P.tabs[A.ftab + r * A.ncols + c];
}
// start of the tensor's buffer.  A.ptr was resolved on the host (souffle_workspace_init): indexing
// the kernel-parameter pointer table at run time goes through the constant cache and misses to L2.
__device__ __forceinline__ char* addr_ptr(const Params& P, const Addr& A) {
  (void)P;
  return (char*)A.ptr - A.base * (A.dtype ? 2 : 4);
}
__device__ __forceinline__ float bf2f(uint16_t b) { return __uint_as_float(((uint32_t)b) << 16); }
__device__ __forceinline__ uint16_t f2bf(float f) {
  __nv_bfloat16 h = __float2bfloat16_rn(f);
  return *reinterpret_cast<uint16_t*>(&h);
}
__device__ __forceinline__ float ld1(const Params& P, const Addr& A, int64_t o) {
  char* p = addr_ptr(P, A);
  if (A.dtype == 0) {
    const float* f = (const float*)p + o;
    return A.cg ? __ldcg(f) : __ldg(f);
  }
  const unsigned short* h = (const unsigned short*)p + o;
  return bf2f(A.cg ? __ldcg(h) : __ldg(h));
}

// load W consecutive-column elements of row r starting at column c0 (nvalid of them)
// element offset of (r, c0) if columns c0 .. c0+W-1 are contiguous in memory, else -1
template <int W>
__device__ __forceinline__ int64_t contig_off(const Params& P, const Addr& A, int64_t r, int64_t c0, int nvalid) {
  if (nvalid != W || W != 8) return -1;
  if (A.mode == 0 && A.cs == 1) return A.base + r * A.rs + c0;
  if (A.mode == 1 && A.cvec && (c0 & (CHUNK - 1)) == 0) return A.base + P.tabs[A.rtab + r] + P.tabs[A.ctab + c0];
  return -1;
}

template <int W>
struct Vec {
  float x[W];
};

// ---- shared-memory tensor cache (§6.5; placement decided on the host by an LRU
// scan, host/lower.cpp tensor_cache).  Every stage that touches a cached tensor is a row-block stage
// with the same rows and row-block size, so the CTA that deposits row r of the tensor is the CTA that
// reads it back; the stages are separated by at least a __syncthreads.
extern __shared__ __align__(1024) char g_dyn_smem[];
__device__ __forceinline__ float* cache_elem(const Addr& A, int64_t r, int64_t c) {
  float* base = reinterpret_cast<float*>((((uintptr_t)g_dyn_smem + 1023) & ~(uintptr_t)1023) + EXEC_SMEM);
  const uint32_t rb = (uint32_t)r / (uint32_t)A.crb;
  const uint32_t it = rb / gridDim.x;
  return base + (A.cache - 1) + ((size_t)it * A.crb + (uint32_t)r - rb * (uint32_t)A.crb) * (size_t)A.rs + (size_t)c * A.cs;
}
template <int W>
__device__ __forceinline__ void cache_ld(const Addr& A, int64_t r, int64_t c0, int nvalid, float* v) {
  const float* q = cache_elem(A, r, c0);
  if (W == 8 && A.cs == 1 && nvalid == 8 && ((uintptr_t)q & 15) == 0) {
    const float4 a = reinterpret_cast<const float4*>(q)[0], b = reinterpret_cast<const float4*>(q)[1];
    v[0] = a.x; v[1 % W] = a.y; v[2 % W] = a.z; v[3 % W] = a.w; v[4 % W] = b.x; v[5 % W] = b.y; v[6 % W] = b.z; v[7 % W] = b.w;
    return;
  }
#pragma unroll
  for (int j = 0; j < W; ++j) v[j] = j < nvalid ? q[(int64_t)j * A.cs] : 0.f;
}
template <int W>
__device__ __forceinline__ void cache_st(const Addr& A, int64_t r, int64_t c0, int nvalid, const float* v) {
  float* q = cache_elem(A, r, c0);
  if (W == 8 && A.cs == 1 && nvalid == 8 && ((uintptr_t)q & 15) == 0) {
    float u[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) u[j] = A.dtype ? __uint_as_float((uint32_t)f2bf(v[j % W]) << 16) : v[j % W];
    reinterpret_cast<float4*>(q)[0] = make_float4(u[0], u[1], u[2], u[3]);
    reinterpret_cast<float4*>(q)[1] = make_float4(u[4], u[5], u[6], u[7]);
    return;
  }
#pragma unroll
  for (int j = 0; j < W; ++j)   // rounded as a global round trip would round it
    if (j < nvalid) q[(int64_t)j * A.cs] = A.dtype ? __uint_as_float((uint32_t)f2bf(v[j]) << 16) : v[j];
}

// The element-access helpers and the unary math exist once each (out of line): with everything
// inlined the kernel was 1.3 MB of SASS and every stage ran from a cold instruction cache.
template <int W>
__device__ __noinline__ Vec<W> ld_vec_impl(const Params& P, const Addr& A, int64_t r, int64_t c0, int nvalid) {
  Vec<W> out;
  float* v = out.x;
  const int64_t o = contig_off<W>(P, A, r, c0, nvalid);
  if (o >= 0) {
    char* p = addr_ptr(P, A);
    if (A.dtype == 0 && (o & 3) == 0) {
      const float4* q = reinterpret_cast<const float4*>((const float*)p + o);
      float4 a = A.cg ? __ldcg(q) : __ldg(q);
      float4 b = A.cg ? __ldcg(q + 1) : __ldg(q + 1);
      v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
      return out;
    }
    if (A.dtype == 1 && (o & 7) == 0) {
      const uint4* q = reinterpret_cast<const uint4*>((const uint16_t*)p + o);
      uint4 a = A.cg ? __ldcg(q) : __ldg(q);
      const uint32_t w[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        v[2 * j] = __uint_as_float(w[j] << 16);
        v[2 * j + 1] = __uint_as_float(w[j] & 0xFFFF0000u);
      }
      return out;
    }
  }
  if (A.mode == 0 && A.cs == 0) {   // broadcast along the row (e.g. per-row statistics)
    float x = ld1(P, A, A.base + r * A.rs);
#pragma unroll
    for (int j = 0; j < W; ++j) v[j] = x;
    return out;
  }
#pragma unroll
  for (int j = 0; j < W; ++j) v[j] = j < nvalid ? ld1(P, A, addr_off(P, A, r, c0 + j)) : 0.f;
  return out;
}

// Inline fast paths (contiguous vector / row broadcast) so that independent loads of a chunk are
// all in flight together; only the generic per-element gather is out of line.
template <int W>
__device__ __forceinline__ void ld_vec_g(const Params& P, const Addr& A, int64_t r, int64_t c0, int nvalid, float* v) {
  const int64_t o = contig_off<W>(P, A, r, c0, nvalid);
  if (W == 8 && o >= 0 && A.dtype == 0 && (o & 3) == 0) {
    const float4* q = reinterpret_cast<const float4*>((const float*)addr_ptr(P, A) + o);
    float4 a = A.cg ? __ldcg(q) : __ldg(q);
    float4 b = A.cg ? __ldcg(q + 1) : __ldg(q + 1);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4 % W] = b.x; v[5 % W] = b.y; v[6 % W] = b.z; v[7 % W] = b.w;
    return;
  }
  if (W == 8 && o >= 0 && A.dtype == 1 && (o & 7) == 0) {
    const uint4* q = reinterpret_cast<const uint4*>((const uint16_t*)addr_ptr(P, A) + o);
    uint4 a = A.cg ? __ldcg(q) : __ldg(q);
    const uint32_t w[4] = {a.x, a.y, a.z, a.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      v[(2 * j) % W] = __uint_as_float(w[j] << 16);
      v[(2 * j + 1) % W] = __uint_as_float(w[j] & 0xFFFF0000u);
    }
    return;
  }
  if (A.mode == 0 && A.cs == 0) {   // broadcast along the row (e.g. per-row statistics)
    float x = ld1(P, A, A.base + r * A.rs);
#pragma unroll
    for (int j = 0; j < W; ++j) v[j] = x;
    return;
  }
  Vec<W> t = ld_vec_impl<W>(P, A, r, c0, nvalid);
#pragma unroll
  for (int j = 0; j < W; ++j) v[j] = t.x[j];
}

// a cached tensor is read from shared memory; a filling load (the tensor's first use in the launch)
// reads global memory and deposits whole chunks (the W = 1 row-start probe of a shifted reduction does not)
template <int W>
__device__ __forceinline__ void ld_vec(const Params& P, const Addr& A, int64_t r, int64_t c0, int nvalid, float* v) {
  if (A.cache && !(A.cmode & CM_FILL)) {
    cache_ld<W>(A, r, c0, nvalid, v);
    return;
  }
  ld_vec_g<W>(P, A, r, c0, nvalid, v);
  if (W == CHUNK && A.cache) cache_st<W>(A, r, c0, nvalid, v);
}

template <int W>
__device__ __noinline__ void st_vec_impl(const Params& P, const Addr& A, int64_t r, int64_t c0, int nvalid,
                                         const Vec<W> vv) {
  const float* v = vv.x;
  char* p = addr_ptr(P, A);
  const int64_t o = contig_off<W>(P, A, r, c0, nvalid);
  if (o >= 0) {
    if (A.dtype == 0 && (o & 3) == 0) {
      float4* q = reinterpret_cast<float4*>((float*)p + o);
      q[0] = make_float4(v[0], v[1], v[2], v[3]);
      q[1] = make_float4(v[4], v[5], v[6], v[7]);
      return;
    }
    if (A.dtype == 1 && (o & 7) == 0) {
      uint4 a;
      a.x = (uint32_t)f2bf(v[0]) | ((uint32_t)f2bf(v[1]) << 16);
      a.y = (uint32_t)f2bf(v[2]) | ((uint32_t)f2bf(v[3]) << 16);
      a.z = (uint32_t)f2bf(v[4]) | ((uint32_t)f2bf(v[5]) << 16);
      a.w = (uint32_t)f2bf(v[6]) | ((uint32_t)f2bf(v[7]) << 16);
      *reinterpret_cast<uint4*>((uint16_t*)p + o) = a;
      return;
    }
  }
#pragma unroll
  for (int j = 0; j < W; ++j) {
    if (j < nvalid) {
      int64_t o = addr_off(P, A, r, c0 + j);
      if (A.dtype == 0) ((float*)p)[o] = v[j];
      else ((uint16_t*)p)[o] = f2bf(v[j]);
    }
  }
}

template <int W>
__device__ __forceinline__ void st_vec(const Params& P, const Addr& A, int64_t r, int64_t c0, int nvalid, const float* v) {
  if (A.cache) {
    cache_st<W>(A, r, c0, nvalid, v);
    if (A.cmode & CM_NOSTORE) return;
  }
  const int64_t o = contig_off<W>(P, A, r, c0, nvalid);
  if (W == 8 && o >= 0 && A.dtype == 0 && (o & 3) == 0) {
    float4* q = reinterpret_cast<float4*>((float*)addr_ptr(P, A) + o);
    q[0] = make_float4(v[0], v[1 % W], v[2 % W], v[3 % W]);
    q[1] = make_float4(v[4 % W], v[5 % W], v[6 % W], v[7 % W]);
    return;
  }
  if (W == 8 && o >= 0 && A.dtype == 1 && (o & 7) == 0) {
    uint4 a;
    a.x = (uint32_t)f2bf(v[0]) | ((uint32_t)f2bf(v[1 % W]) << 16);
    a.y = (uint32_t)f2bf(v[2 % W]) | ((uint32_t)f2bf(v[3 % W]) << 16);
    a.z = (uint32_t)f2bf(v[4 % W]) | ((uint32_t)f2bf(v[5 % W]) << 16);
    a.w = (uint32_t)f2bf(v[6 % W]) | ((uint32_t)f2bf(v[7 % W]) << 16);
    *reinterpret_cast<uint4*>((uint16_t*)addr_ptr(P, A) + o) = a;
    return;
  }
  Vec<W> t;
#pragma unroll
  for (int j = 0; j < W; ++j) t.x[j] = v[j];
  st_vec_impl<W>(P, A, r, c0, nvalid, t);
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
template <int W, class F>
__device__ __forceinline__ void with_pf(float (&pf)[kMaxPf][W], int s, F f) {
  switch (s) {
    case 0: f(pf[0]); break;
    case 1: f(pf[1]); break;
    case 2: f(pf[2]); break;
    case 3: f(pf[3]); break;
    case 4: f(pf[4]); break;
    default: f(pf[5]); break;
  }
}

__device__ __forceinline__ bool is_load(int op) { return op == OP_LOAD || op == OP_BINL; }

template <int W>
__device__ __noinline__ Vec<W> vec_un_impl(int fn, Vec<W> v) {
  float* x = v.x;
  switch (fn) {
    case FN_EXP:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = expf(x[j]);
      break;
    case FN_TANH:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = tanhf(x[j]);
      break;
    case FN_SIGMOID:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = 1.f / (1.f + expf(-x[j]));
      break;
    case FN_RELU:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = fmaxf(x[j], 0.f);
      break;
    case FN_GELU:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = 0.5f * x[j] * (1.f + erff(x[j] * 0.70710678118654752f));
      break;
    case FN_RSQRT:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = rsqrtf(x[j]);
      break;
    case FN_NEG:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = -x[j];
      break;
  }
  return v;
}
template <int W>
__device__ __forceinline__ void vec_un(int fn, float* x) {
  Vec<W> t;
#pragma unroll
  for (int j = 0; j < W; ++j) t.x[j] = x[j];
  t = vec_un_impl<W>(fn, t);
#pragma unroll
  for (int j = 0; j < W; ++j) x[j] = t.x[j];
}
// x = fn(x, y)
template <int W>
__device__ __forceinline__ void vec_bin(int fn, float* x, const float* y) {
  switch (fn) {
    case FN_ADD:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] += y[j];
      break;
    case FN_SUB:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] -= y[j];
      break;
    case FN_MUL:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] *= y[j];
      break;
    case FN_DIV:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = x[j] / y[j];
      break;
    case FN_MAX:
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = fmaxf(x[j], y[j]);
      break;
  }
}

struct Red4 {
  float x[MAX_RED];
};
template <int W>
struct ProgOut {
  Vec<W> r0;
  Red4 red;
};

// Runs a fused-chain program at domain row r, columns c0 .. c0+nvalid-1.  acc = accumulator
// values of those columns.  Row reductions accumulate into red (returned; caller flushes).
// Returns register 0 as well (reduction pre-programs).  Not inlined (one copy of the
// interpreter per width); everything is passed by value so nothing lives on the stack -- local
// memory is expensive here because every grid barrier's acquire invalidates L1.
template <int W>
__device__ __noinline__ ProgOut<W> run_prog_impl(const Params& P, const Prog G, int64_t r, int64_t c0, int nvalid,
                                                 const Vec<W> accv, Red4 redin) {
  const float* acc = accv.x;
  ProgOut<W> out;
  float* out0 = out.r0.x;
  float* red = redin.x;
  // ---- pass 1: issue the first kMaxPf loads of the program as one batch
  float pf[kMaxPf][W];
  {
    int i = 0;
#pragma unroll
    for (int s = 0; s < kMaxPf; ++s) {
      while (i < G.len && !is_load(G.ins[i].op)) ++i;
      if (i < G.len) {
        ld_vec<W>(P, G.addr[G.ins[i].addr], r, c0, nvalid, pf[s]);
        ++i;
      }
    }
  }
  // ---- pass 2: execute
  Regs<W> R;
#pragma unroll
  for (int k = 0; k < NREG; ++k)
#pragma unroll
    for (int j = 0; j < W; ++j) R.v[k][j] = 0.f;
  // every interpreted op works on whole W-wide vectors; the op / function switches are taken
  // once per vector (never inside the lane loop)
  int ls = 0;
  for (int i = 0; i < G.len; ++i) {
    const Ins I = G.ins[i];
    float x[W], t[W];
    with_reg<W>(R, I.a, [&](float* y) {
#pragma unroll
      for (int j = 0; j < W; ++j) x[j] = y[j];
    });
    const int op = I.op;
    if (op == OP_LOAD || op == OP_BINL) {
      if (ls < kMaxPf) {
        with_pf<W>(pf, ls, [&](float* y) {
#pragma unroll
          for (int j = 0; j < W; ++j) t[j] = y[j];
        });
      } else {
        ld_vec<W>(P, G.addr[I.addr], r, c0, nvalid, t);
      }
      ++ls;
    } else if (op == OP_BIN || op == OP_BINR || op == OP_MOV) {
      with_reg<W>(R, I.b, [&](float* y) {
#pragma unroll
        for (int j = 0; j < W; ++j) t[j] = y[j];
      });
    }
    const bool swap = (op == OP_BINR) || (op == OP_BINL && I.b);
    if (swap) {   // x = fn(t, x): exchange the operands, then apply fn(x, t)
#pragma unroll
      for (int j = 0; j < W; ++j) {
        float u = x[j];
        x[j] = t[j];
        t[j] = u;
      }
    }
    switch (op) {
      case OP_LOAD:
      case OP_MOV:
#pragma unroll
        for (int j = 0; j < W; ++j) x[j] = t[j];
        break;
      case OP_ACC:
#pragma unroll
        for (int j = 0; j < W; ++j) x[j] = acc[j];
        break;
      case OP_UN: vec_un<W>(I.fn, x); break;
      case OP_SCAL:
        if (I.fn == FN_ADDS) {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] += I.imm;
        } else {
#pragma unroll
          for (int j = 0; j < W; ++j) x[j] *= I.imm;
        }
        break;
      case OP_BIN:
      case OP_BINR:
      case OP_BINL: vec_bin<W>(I.fn, x, t); break;
      case OP_STORE: st_vec<W>(P, G.addr[I.addr], r, c0, nvalid, x); continue;
      case OP_RED: {
        float s = 0.f;
#pragma unroll
        for (int j = 0; j < W; ++j)
          if (j < nvalid) s += x[j];
        s *= I.imm;
        switch (I.b) {   // compile-time indices keep red[] in registers
          case 0: red[0] += s; break;
          case 1: red[1] += s; break;
          case 2: red[2] += s; break;
          default: red[3] += s; break;
        }
        continue;
      }
    }
    with_reg<W>(R, I.a, [&](float* y) {
#pragma unroll
      for (int j = 0; j < W; ++j) y[j] = x[j];
    });
  }
#pragma unroll
  for (int j = 0; j < W; ++j) out0[j] = R.v[0][j];
#pragma unroll
  for (int k = 0; k < MAX_RED; ++k) out.red.x[k] = red[k];
  return out;
}

__device__ __forceinline__ void red_add(Red4& red, int slot, float s) {
  switch (slot) {
    case 0: red.x[0] += s; break;
    case 1: red.x[1] += s; break;
    case 2: red.x[2] += s; break;
    default: red.x[3] += s; break;
  }
}

// Compiled fast paths (FastPath kinds 1 and 2): straight-line code, all loads issued first.
template <int W>
__device__ __noinline__ Red4 run_fast(const Params& P, const Prog G, int64_t r, int64_t c0, int nvalid,
                                      const Vec<W> accv, Red4 red) {
  const FastPath& f = *G.fast;
  float v[W];
  if (f.kind == 1) {
    float s0[W], s1[W];
    if (f.side0 >= 0) ld_vec<W>(P, G.addr[G.ins[f.side0].addr], r, c0, nvalid, s0);
    if (f.side1 >= 0) ld_vec<W>(P, G.addr[G.ins[f.side1].addr], r, c0, nvalid, s1);
#pragma unroll
    for (int j = 0; j < W; ++j) v[j] = accv.x[j];
    if (f.side0 >= 0) {
#pragma unroll
      for (int j = 0; j < W; ++j) v[j] += s0[j];
    }
    if (f.side1 >= 0) {
#pragma unroll
      for (int j = 0; j < W; ++j) v[j] += s1[j];
    }
    if (f.act >= 0) vec_un<W>(f.act, v);
  } else {
    float x[W], mu[W], ms[W], g[W], b[W];
    ld_vec<W>(P, G.addr[G.ins[f.ln_x].addr], r, c0, nvalid, x);
    ld_vec<W>(P, G.addr[G.ins[f.ln_mu].addr], r, c0, nvalid, mu);
    ld_vec<W>(P, G.addr[G.ins[f.ln_msq].addr], r, c0, nvalid, ms);
    ld_vec<W>(P, G.addr[G.ins[f.ln_g].addr], r, c0, nvalid, g);
    ld_vec<W>(P, G.addr[G.ins[f.ln_b].addr], r, c0, nvalid, b);
#pragma unroll
    for (int j = 0; j < W; ++j) {
      const float m = mu[j];
      const float rs = rsqrtf((ms[j] - m * m) + f.eps);
      v[j] = ((x[j] - m) * rs) * g[j] + b[j];
    }
  }
  if (f.st0 >= 0) st_vec<W>(P, G.addr[G.ins[f.st0].addr], r, c0, nvalid, v);
  if (f.st1 >= 0) st_vec<W>(P, G.addr[G.ins[f.st1].addr], r, c0, nvalid, v);
  if (f.red_sum >= 0) {
    float s = 0.f;
#pragma unroll
    for (int j = 0; j < W; ++j)
      if (j < nvalid) s += v[j];
    red_add(red, G.ins[f.red_sum].b, s * f.red_scale_sum);
  }
  if (f.red_sq >= 0) {
    float s = 0.f;
#pragma unroll
    for (int j = 0; j < W; ++j)
      if (j < nvalid) s += v[j] * v[j];
    red_add(red, G.ins[f.red_sq].b, s * f.red_scale_sq);
  }
  return red;
}

// Inline wrapper; `red` must be a register array with compile-time indexing at the call site.
template <int W>
__device__ __forceinline__ void run_prog(const Params& P, const Prog& G, int64_t r, int64_t c0, int nvalid,
                                         const float* acc, float* red, float* out0 = nullptr) {
  Vec<W> a;
#pragma unroll
  for (int j = 0; j < W; ++j) a.x[j] = acc[j];
  Red4 ri;
#pragma unroll
  for (int k = 0; k < MAX_RED; ++k) ri.x[k] = red[k];
  if (!out0 && G.fast->kind != 0) {
    Red4 ro = run_fast<W>(P, G, r, c0, nvalid, a, ri);
#pragma unroll
    for (int k = 0; k < MAX_RED; ++k) red[k] = ro.x[k];
    return;
  }
  ProgOut<W> o = run_prog_impl<W>(P, G, r, c0, nvalid, a, ri);
#pragma unroll
  for (int k = 0; k < MAX_RED; ++k) red[k] = o.red.x[k];
  if (out0) {
#pragma unroll
    for (int j = 0; j < W; ++j) out0[j] = o.r0.x[j];
  }
}

// flush per-thread partial row reductions (one atomic per row and reduction, §6.3)
__device__ __forceinline__ void flush_reds(const Params& P, const Prog& G, int64_t r, float* red) {
  for (int i = 0; i < G.len; ++i) {
    const Ins I = G.ins[i];
    if (I.op != OP_RED) continue;
    const Addr& A = G.addr[I.addr];
    float* p = (float*)addr_ptr(P, A) + addr_off(P, A, r, 0);
    float v = I.b == 0 ? red[0] : I.b == 1 ? red[1] : I.b == 2 ? red[2] : red[3];
    atomicAdd(p, v);
  }
#pragma unroll
  for (int k = 0; k < MAX_RED; ++k) red[k] = 0.f;
}

__device__ __forceinline__ void progress(const Params& P, int stage, int point) {
  if (threadIdx.x == 0 && blockIdx.x < 256) *(volatile unsigned*)&P.progress[blockIdx.x] = ((unsigned)stage << 8) | (unsigned)point;
}

// ================================================================== grid barrier
// Split-phase barrier on a monotonically increasing counter.  arrive: all threads order their
// global writes (generic proxy) before the async proxy (TMA) of other CTAs, the CTA synchronises,
// one thread performs a release-add.  wait: that thread spins with acquire loads, then the CTA
// synchronises.  Between the two the CTA prefetches the next stage's static data.
__device__ __forceinline__ void barrier_arrive(const Params& P, unsigned& nb, const SmemCtrl* ctl) {
  ptx::fence_proxy_async();
  __syncthreads();
  ++nb;
  if (threadIdx.x == 0) {
    unsigned old;
    asm volatile("atom.release.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(&P.ctrl[0]) : "memory");
    if (P.prof && old == nb * gridDim.x - 1) {   // last CTA to arrive: end of the stage's critical path
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      P.prof[P.n_stages_total + 1 + 8 * ctl->cur_stage + 7] = t;
    }
  }
}
__device__ __forceinline__ void barrier_wait(const Params& P, unsigned nb) {
  if (threadIdx.x == 0) {
    const unsigned target = nb * gridDim.x;
    // relaxed polling with back-off (idle CTAs must not flood L2 while others work), then one
    // acquire fence
    unsigned v;
    unsigned long long t0 = 0;
    for (uint32_t n = 0;; ++n) {
      asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&P.ctrl[0]) : "memory");
      if (v >= target) break;
      __nanosleep(64);
      if ((n & 1023u) == 1023u) {   // watchdog: a dependency that never resolves aborts the launch
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        if (t0 == 0) t0 = t;
        else if (t - t0 > 3000000000ull) {
          printf("souffle_exec_kernel: grid barrier %u timed out in CTA %d (count %u of %u)\n", nb, (int)blockIdx.x,
                 v, target);
          const unsigned mine = *(volatile unsigned*)&P.progress[blockIdx.x];
          for (int c = 0; c < (int)gridDim.x && c < 256; ++c) {
            const unsigned pc = *(volatile unsigned*)&P.progress[c];
            if ((pc >> 8) < (mine >> 8)) printf("  lagging CTA %d: stage %u point %u\n", c, pc >> 8, pc & 255u);
          }
          __trap();
        }
      }
    }
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
  }
  __syncthreads();
}

__device__ __forceinline__ Prog cached_prog(char* smem, int k) { return cache_of(smem, k)->p; }

// Stage s's descriptor, and the program(s) and member record of this CTA's first task -> smem.
__device__ void prefetch_stage(const Params& P, int s, char* smem) {
  SmemCtrl* ctl = ctrl_of(smem);
  Stage* sst = stage_of(smem);
  if (threadIdx.x < (int)(sizeof(Stage) / 16))
    reinterpret_cast<int4*>(sst)[threadIdx.x] = __ldg(reinterpret_cast<const int4*>(P.stages + s) + threadIdx.x);
  if (threadIdx.x == 0) ctl->pf_member = 0;
  __syncthreads();
  const int kind = sst->kind;
  if (kind == ST_EW || kind == ST_ATTN) {
    stage_prog(P, sst->prog, cache_of(smem, 0));
  } else if (kind == ST_REDUCE) {
    stage_prog(P, sst->prog, cache_of(smem, 0));
    stage_prog(P, sst->post, cache_of(smem, 1));
  } else {
    const int task = blockIdx.x;
    const int t = threadIdx.x;
    if (t >= 1 && t < sst->nmem && task < sst->ntasks && __ldg(&P.members[sst->mem0 + t].task0) <= task)
      atomicMax(&ctl->pf_member, t);
    __syncthreads();
    const int mi = ctl->pf_member;
    if (t < (int)(sizeof(GemmMember) / 4))
      reinterpret_cast<int*>(&ctl->mem)[t] = __ldg(reinterpret_cast<const int*>(P.members + sst->mem0 + mi) + t);
    __syncthreads();
    stage_prog(P, ctl->mem.prog, cache_of(smem, 0));
  }
}

// ================================================================== EW stage
__device__ __noinline__ void run_ew(const Params& P, const Stage& st, char* smem) {
  const Prog G = cached_prog(smem, 0);
  if (threadIdx.x == 0) mark(P, ctrl_of(smem), 0);   // program staged
  const int64_t cpr = (st.cols + CHUNK - 1) / CHUNK;
  const int64_t total = (int64_t)st.rows * cpr;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  if (st.rblk > 0) {   // row-block ownership (CTA-local dependencies with the launch's REDUCE stages)
    const int64_t per = (int64_t)st.rblk * cpr;
    for (int64_t rb = blockIdx.x; rb * st.rblk < st.rows; rb += gridDim.x) {
      const int64_t n = min(per, total - rb * per);
      for (int64_t i = threadIdx.x; i < n; i += kThreads) {
        const int64_t t = rb * per + i;
        const int64_t r = t / cpr, c0 = (t % cpr) * CHUNK;
        const int nv = (int)((st.cols - c0) < CHUNK ? (st.cols - c0) : CHUNK);
        float acc[CHUNK] = {0, 0, 0, 0, 0, 0, 0, 0};
        run_prog<CHUNK>(P, G, r, c0, nv, acc, red);
        flush_reds(P, G, r, red);
      }
    }
    __syncthreads();
    if (threadIdx.x == 0) mark(P, ctrl_of(smem), 2);
    return;
  }
  for (int64_t t = (int64_t)blockIdx.x * kThreads + threadIdx.x; t < total; t += (int64_t)gridDim.x * kThreads) {
    int64_t r = t / cpr;
    int64_t c0 = (t % cpr) * CHUNK;
    int nv = (int)((st.cols - c0) < CHUNK ? (st.cols - c0) : CHUNK);
    float acc[CHUNK] = {0, 0, 0, 0, 0, 0, 0, 0};
    if (t == 0) mark(P, ctrl_of(smem), 3);   // before the chain (thread 0 of CTA 0)
    run_prog<CHUNK>(P, G, r, c0, nv, acc, red);
    if (t == 0) mark(P, ctrl_of(smem), 4);   // after the chain
    flush_reds(P, G, r, red);
    if (t == 0) mark(P, ctrl_of(smem), 1);   // first chunk done (thread 0 of CTA 0)
  }
  __syncthreads();
  if (threadIdx.x == 0) mark(P, ctrl_of(smem), 2);   // all chunks of this CTA done
}

// ================================================================== REDUCE stage (warp per row)
// Rows of at most 16 chunks (<= 128 columns, e.g. the 49-wide window-attention softmax rows of Swin)
// are packed several per warp: a group of G lanes (a power of two >= the row's chunk count) owns one
// row, so short rows do not leave most of the warp idle.
__device__ __noinline__ void run_reduce(const Params& P, const Stage& st, char* smem) {
  const Prog pre = cached_prog(smem, 0);
  const Prog post = cached_prog(smem, 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  // the host fixed the row-block size (Stage.rblk = 8 warps x 32/G rows, G = lanes per row)
  const int rpw = st.rblk / 8;                 // rows per warp
  const int G = 32 / rpw;
  const int sub = lane / G, gl = lane % G;     // row slot within the warp, lane within the group
  const int64_t rows_per_cta = 8 * rpw;
  for (int64_t ob = (int64_t)blockIdx.x * rows_per_cta + warp * rpw; ob < st.rows; ob += (int64_t)gridDim.x * rows_per_cta) {
    const int64_t o = ob + sub;
    const bool live = o < st.rows;
    float acc = st.red_fn ? -INFINITY : 0.f;
    // a mean (sum with scale 1/E) is accumulated relative to the row's first element v0 and
    // returned as v0 + scale * sum(v - v0): exact for a constant row, no loss of the small spread
    // of an offset row (the LayerNorm mean, then x - mean, must be exactly 0 for a constant row)
    const bool shifted = st.red_fn == 0 && st.red_scale != 1.f;
    float v0 = 0.f;
    if (live && shifted) {
      float z1[1] = {0.f}, d1[MAX_RED] = {0.f, 0.f, 0.f, 0.f}, e1[1];
      run_prog<1>(P, pre, o, 0, 1, z1, d1, e1);
      v0 = e1[0];
    }
    if (live) {
      for (int64_t c0 = (int64_t)gl * CHUNK; c0 < st.cols; c0 += (int64_t)G * CHUNK) {
        int nv = (int)((st.cols - c0) < CHUNK ? (st.cols - c0) : CHUNK);
        float vals[CHUNK];
        float zero[CHUNK] = {0, 0, 0, 0, 0, 0, 0, 0};
        float dummy[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
        run_prog<CHUNK>(P, pre, o, c0, nv, zero, dummy, vals);
#pragma unroll
        for (int j = 0; j < CHUNK; ++j)
          if (j < nv) acc = st.red_fn ? fmaxf(acc, vals[j]) : acc + (vals[j] - v0);
      }
    }
    for (int s2 = G >> 1; s2 > 0; s2 >>= 1) {
      float y = __shfl_xor_sync(0xffffffffu, acc, s2);
      acc = st.red_fn ? fmaxf(acc, y) : acc + y;
    }
    acc = shifted ? v0 + acc * st.red_scale : acc * st.red_scale;
    if (live && gl == 0) {
      float a1[1] = {acc};
      run_prog<1>(P, post, o, 0, 1, a1, red);
      flush_reds(P, post, o, red);
    }
  }
}

// ================================================================== SIMT GEMM stage
__device__ __noinline__ void run_gemm_simt(const Params& P, const Stage& st, char* smem) {
  char* ring = smem + kCtrlBytes;
  float(*As)[68] = reinterpret_cast<float(*)[68]>(ring);
  float(*Bs)[68] = reinterpret_cast<float(*)[68]>(ring + 16 * 68 * 4);
  const int tid = threadIdx.x, ty = tid >> 3, tx = tid & 7;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  const int pf = ctrl_of(smem)->pf_member;   // prefetched member (program in cache 0)
  int cur = pf;
  Prog G = cached_prog(smem, 0);
  for (int task = blockIdx.x; task < st.ntasks; task += gridDim.x) {
    int mi = pf;
    if (task != (int)blockIdx.x) {
      mi = 0;
      while (mi + 1 < st.nmem && P.members[st.mem0 + mi + 1].task0 <= task) ++mi;
    }
    const GemmMember& M = (mi == pf) ? ctrl_of(smem)->mem : P.members[st.mem0 + mi];
    if (mi != cur) {
      __syncthreads();   // every warp is done with the previous member's program before it is replaced
      G = stage_prog(P, M.prog, cache_of(smem, 0));
      cur = mi;
    }
    const int local = task - M.task0;
    if (M.gemv) {
      // skinny GEMM (e.g. a classifier head on one pooled row): warp w computes output 8 * task + w,
      // lanes stride over K (coalesced rows of B), shuffle reduction, lane 0 runs the chain
      const Addr A = P.addrs[M.a_addr];
      const Addr B = P.addrs[M.b_addr];
      const int warp = tid >> 5, lane = tid & 31;
      const int64_t rows = (int64_t)M.batch * M.M;
      for (int i = 0; i < 1; ++i) {
        const int64_t idx = (int64_t)local * 8 + warp;
        const int64_t r = idx / M.N;
        const int n = (int)(idx % M.N);
        if (r >= rows) break;
        const int64_t b = r / M.M;
        float acc = 0.f;
        for (int k = lane; k < M.K; k += 32) {
          float a = ld1(P, A, addr_off(P, A, r, k));
          float bb = ld1(P, B, addr_off(P, B, b * M.N + n, k));
          if (M.prec) {
            a = __bfloat162float(__float2bfloat16_rn(a));
            bb = __bfloat162float(__float2bfloat16_rn(bb));
          }
          acc = fmaf(a, bb, acc);
        }
#pragma unroll
        for (int s2 = 16; s2 > 0; s2 >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, s2);
        if (lane == 0) {
          float a1[1] = {acc};
          run_prog<1>(P, G, r, n, 1, a1, red);
          flush_reds(P, G, r, red);
        }
      }
      continue;
    }
    // split-K (few tiles, long K): task = (tile, split); split s accumulates K range [s k_split, ...)
    const int split = M.splits > 1 ? local % M.splits : 0;
    const int tl = M.splits > 1 ? local / M.splits : local;
    const int tmi = tl / M.tiles_n, tn = tl % M.tiles_n;
    const int mt = (M.M + 63) / 64;
    const int b = tmi / mt, tm = tmi % mt;
    const Addr A = P.addrs[M.a_addr];
    const Addr B = P.addrs[M.b_addr];
    const int kbeg = M.splits > 1 ? split * M.k_split : 0;
    const int kend = M.splits > 1 ? min(M.K, kbeg + M.k_split) : M.K;
    float acc[2][8];
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
    for (int k0 = kbeg; k0 < kend; k0 += 16) {
      __syncthreads();
      float av[4], bv[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        int e = tid + q * kThreads;
        int kk = e >> 6, i = e & 63;
        int m = tm * 64 + i, n = tn * 64 + i, k = k0 + kk;
        av[q] = (m < M.M && k < kend) ? ld1(P, A, addr_off(P, A, (int64_t)b * M.M + m, k)) : 0.f;
        bv[q] = (n < M.N && k < kend) ? ld1(P, B, addr_off(P, B, (int64_t)b * M.N + n, k)) : 0.f;
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        int e = tid + q * kThreads;
        int kk = e >> 6, i = e & 63;
        float a = av[q], bb = bv[q];
        if (M.prec) {
          a = __bfloat162float(__float2bfloat16_rn(a));
          bb = __bfloat162float(__float2bfloat16_rn(bb));
        }
        As[kk][i] = a;
        Bs[kk][i] = bb;
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < 16; ++kk) {
        float a0 = As[kk][ty * 2], a1 = As[kk][ty * 2 + 1];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          float bvv = Bs[kk][tx * 8 + j];
          acc[0][j] = fmaf(a0, bvv, acc[0][j]);
          acc[1][j] = fmaf(a1, bvv, acc[1][j]);
        }
      }
    }
    if (M.splits > 1) {
      // partials into the fp32 tile accumulator (vector reductions into L2); the last split to arrive
      // (per-tile counter) runs the fused chain on the sum and re-zeroes the tile
      float* accbuf = (float*)P.ws_data + M.acc_off + (int64_t)tl * 64 * 64;
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        float* p = accbuf + (ty * 2 + i) * 64 + tx * 8;
        asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(acc[i][0]), "f"(acc[i][1]),
                     "f"(acc[i][2]), "f"(acc[i][3]) : "memory");
        asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p + 4), "f"(acc[i][4]), "f"(acc[i][5]),
                     "f"(acc[i][6]), "f"(acc[i][7]) : "memory");
      }
      __syncthreads();
      SmemCtrl* ctl = ctrl_of(smem);
      if (threadIdx.x == 0) {
        unsigned* cnt = (unsigned*)P.ws_data + M.cnt_off + tl;
        unsigned old;
        asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(cnt) : "memory");
        ctl->flag = (old == (unsigned)(M.splits - 1)) ? 1 : 0;
        if (ctl->flag) *cnt = 0u;   // self-cleaning for the next run
      }
      __syncthreads();
      const bool last = ctl->flag != 0;
      __syncthreads();   // the flag is read by every thread before the next task may rewrite it
      if (!last) continue;
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        float4* p = reinterpret_cast<float4*>(accbuf + (ty * 2 + i) * 64 + tx * 8);
        const float4 a0 = __ldcg(p), a1 = __ldcg(p + 1);
        __stcg(p, make_float4(0.f, 0.f, 0.f, 0.f));
        __stcg(p + 1, make_float4(0.f, 0.f, 0.f, 0.f));
        acc[i][0] = a0.x; acc[i][1] = a0.y; acc[i][2] = a0.z; acc[i][3] = a0.w;
        acc[i][4] = a1.x; acc[i][5] = a1.y; acc[i][6] = a1.z; acc[i][7] = a1.w;
      }
    }
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      int m = tm * 64 + ty * 2 + i;
      int c0 = tn * 64 + tx * 8;
      if (m < M.M && c0 < M.N) {
        int nv = min(8, M.N - c0);
        int64_t r = (int64_t)b * M.M + m;
        run_prog<CHUNK>(P, G, r, c0, nv, acc[i], red);
        flush_reds(P, G, r, red);
      }
    }
  }
  __syncthreads();
}

// ================================================================== TC GEMM stage
// swizzled (128B) byte offset of element (row, k-byte) inside a K-major tile with 64-element rows
__device__ __forceinline__ uint32_t sw128(int row, int kbyte) {
  return (uint32_t)(row * 128 + ((((kbyte >> 4) ^ (row & 7)) & 7) << 4) + (kbyte & 15));
}

// Epilogue of one 128 x NT tile (COLS = NT/2 columns per thread).  splits == 1: the fused chain
// runs straight from TMEM.  splits > 1: partials are added into an fp32 tile accumulator with
// vector atomics; the last CTA to arrive (per-tile counter) runs the chain and re-zeroes the tile.
// Runtime loops over 8-column chunks keep only ~8 accumulator registers live (no spills).
__device__ __forceinline__ void tc_epilogue(const Params& P, const Prog& G, const GemmMember& M, SmemCtrl* ctl,
                                            int tile, int m0, int n0, int rows, float* red) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int q = warp & 3, half = warp >> 2;
  const int row = q * 32 + lane;
  const int64_t r = m0 + row;
  const int NT = M.n_tile;
  const int COLS = NT / 2;
  const int cbase = half * COLS;
  const uint32_t taddr = ctl->tmem_base + ((uint32_t)(q * 32) << 16) + cbase;
  if (M.splits == 1) {
#pragma unroll 1
    for (int c = 0; c < COLS; c += 8) {
      float v[8];
      ptx::tmem_ld8(taddr + c, v);
      if (r < rows) run_prog<CHUNK>(P, G, r, n0 + cbase + c, 8, v, red);
    }
    ptx::tc_fence_before();
    if (r < rows) flush_reds(P, G, r, red);
    return;
  }
  float* accbuf = (float*)P.ws_data + M.acc_off + (int64_t)tile * 128 * NT + (int64_t)row * NT + cbase;
#pragma unroll 1
  for (int c = 0; c < COLS; c += 8) {
    float v[8];
    ptx::tmem_ld8(taddr + c, v);
    if (r < rows) {   // fire-and-forget vector reductions into L2
      asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(accbuf + c), "f"(v[0]), "f"(v[1]),
                   "f"(v[2]), "f"(v[3])
                   : "memory");
      asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(accbuf + c + 4), "f"(v[4]), "f"(v[5]),
                   "f"(v[6]), "f"(v[7])
                   : "memory");
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) {
    // acq_rel RMW: releases this CTA's partials (ordered by the CTA barrier), acquires the others'
    unsigned* cnt = (unsigned*)P.ws_data + M.cnt_off + tile;
    unsigned old;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(cnt) : "memory");
    ctl->flag = (old == (unsigned)(M.splits - 1)) ? 1 : 0;
    if (ctl->flag) *cnt = 0u;   // self-cleaning for the next run
  }
  __syncthreads();
  if (threadIdx.x == 128) mark(P, ctl, 3);      // partials added
  if (!ctl->flag) return;
  if (r < rows) {
    // double-buffered: the next chunk's partial sums are in flight while this chunk is processed
    float4 a0 = __ldcg(reinterpret_cast<const float4*>(accbuf));
    float4 a1 = __ldcg(reinterpret_cast<const float4*>(accbuf + 4));
#pragma unroll 1
    for (int c = 0; c < COLS; c += 8) {
      float v[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
      if (c + 8 < COLS) {
        a0 = __ldcg(reinterpret_cast<const float4*>(accbuf + c + 8));
        a1 = __ldcg(reinterpret_cast<const float4*>(accbuf + c + 12));
      }
      __stcg(reinterpret_cast<float4*>(accbuf + c), make_float4(0.f, 0.f, 0.f, 0.f));
      __stcg(reinterpret_cast<float4*>(accbuf + c + 4), make_float4(0.f, 0.f, 0.f, 0.f));
      run_prog<CHUNK>(P, G, r, n0 + cbase + c, 8, v, red);
    }
    flush_reds(P, G, r, red);
  }
  if (threadIdx.x == 128) mark(P, ctl, 4);      // last-arriver epilogue done
}

__device__ __noinline__ void run_gemm_tc(const Params& P, const Stage& st, char* smem) {
  SmemCtrl* ctl = ctrl_of(smem);
  TcState ts = ctl->ts;   // identical in every thread; written back at the end
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  char* ring = smem + kCtrlBytes;
  const char* tmaps = (const char*)P.tmaps;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  const int pf = ctrl_of(smem)->pf_member;   // prefetched member (program in cache 0)
  int cur = pf;
  Prog G = cached_prog(smem, 0);
  for (int task = blockIdx.x; task < st.ntasks; task += gridDim.x) {
    int mi = pf;
    if (task != (int)blockIdx.x) {
      mi = 0;
      while (mi + 1 < st.nmem && P.members[st.mem0 + mi + 1].task0 <= task) ++mi;
    }
    const GemmMember& M = (mi == pf) ? ctrl_of(smem)->mem : P.members[st.mem0 + mi];
    if (mi != cur) {
      __syncthreads();   // every warp is done with the previous member's program before it is replaced
      G = stage_prog(P, M.prog, cache_of(smem, 0));
      cur = mi;
    }
    if (threadIdx.x == 0) mark(P, ctl, 0);      // task start (program staged)
    const int local = task - M.task0;
    const int split = local % M.splits;
    const int tile = local / M.splits;
    const int tm = tile / M.tiles_n, tn = tile % M.tiles_n;
    const int NT = M.n_tile;
    const int rows = M.M * M.batch;
    const int m0 = tm * 128, n0 = tn * NT;
    const int kbeg = split * M.k_split;
    const int kend = min(M.K, kbeg + M.k_split);
    const int nk = (kend - kbeg) / 64;
    const uint32_t a_bytes = 128 * 128, b_bytes = (uint32_t)NT * 128;
    const bool tma_a = M.a_tmap >= 0;

    if (warp == 0 || (!tma_a && (warp == 2 || warp == 3))) {
      // ---------------- producer: TMA B (+A), or manual fp32 -> bf16 A staging by warps 2-3
      for (int i = 0; i < nk; ++i) {
        const uint32_t slot = ts.it_p % kSlots, ph = (ts.it_p / kSlots) & 1;
        char* sa = ring + slot * kSlotBytes;
        char* sb = sa + 16384;
        if (lane == 0) ptx::mbar_wait_wd(&ctl->empty[slot], ph ^ 1);
        __syncwarp();
        if (!tma_a) {
          if (warp != 0) {
            const Addr& A = P.addrs[M.a_f32];
            const float* ap = (const float*)addr_ptr(P, A) + A.base;
            const int t = (warp - 2) * 32 + lane;     // 64 loader threads
#pragma unroll 4
            for (int e = t; e < 128 * 16; e += 64) {  // 128 rows x 16 float4 groups
              int row = e >> 4, g4 = e & 15;
              int m = m0 + row, k = kbeg + i * 64 + g4 * 4;
              float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
              if (m < rows) {
                const float4* q = reinterpret_cast<const float4*>(ap + (int64_t)m * A.rs + k);
                v = A.cg ? __ldcg(q) : __ldg(q);
              }
              uint32_t lo = (uint32_t)f2bf(v.x) | ((uint32_t)f2bf(v.y) << 16);
              uint32_t hi = (uint32_t)f2bf(v.z) | ((uint32_t)f2bf(v.w) << 16);
              *reinterpret_cast<uint2*>(sa + sw128(row, g4 * 8)) = make_uint2(lo, hi);
            }
            ptx::fence_proxy_async();
          }
          asm volatile("bar.sync 2, 96;" ::: "memory");   // warps 0, 2, 3
        }
        if (warp == 0 && lane == 0) {
          ptx::mbar_arrive_expect_tx(&ctl->full[slot], (tma_a ? a_bytes : 0) + b_bytes);
          if (tma_a) ptx::tma_load_2d(sa, tmaps + 128 * M.a_tmap, &ctl->full[slot], kbeg + i * 64, m0);
          ptx::tma_load_2d(sb, tmaps + 128 * M.b_tmap, &ctl->full[slot], kbeg + i * 64, n0);
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
          ptx::mbar_wait_wd(&ctl->full[slot], ph);
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
    }
    // keep the other roles' ring counters in sync (every thread tracks them uniformly)
    if (!(warp == 0 || (!tma_a && (warp == 2 || warp == 3)))) ts.it_p += nk;
    if (warp != 1) ts.it_c += nk;

    // ---------------- epilogue: all 8 warps; warp w reads TMEM lanes 32*(w%4), column half w/4
    if (threadIdx.x == 0) mark(P, ctl, 1);      // producer done issuing
    progress(P, ctl->cur_stage, 1);
    ptx::mbar_wait_wd(&ctl->accb, ts.acc_phase);
    ptx::tc_fence_after();
    if (threadIdx.x == 128) mark(P, ctl, 2);    // accumulator ready
    progress(P, ctl->cur_stage, 2);
    tc_epilogue(P, G, M, ctl, tile, m0, n0, rows, red);
    progress(P, ctl->cur_stage, 3);
    ts.acc_phase ^= 1;
    __syncthreads();
    progress(P, ctl->cur_stage, 4);
  }
  if (threadIdx.x == 0) ctl->ts = ts;
  __syncthreads();
}

// ================================================================== ATTN stage
__device__ __forceinline__ void attn_epilogue(const Params& P, const Prog& G, SmemCtrl* ctl, int b, int S, int d,
                                              float* red) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int q = warp & 3, half = warp >> 2;
  const int row = q * 32 + lane;
  const int COLS = d / 2;
  const uint32_t taddr = ctl->tmem_base + 128 + ((uint32_t)(q * 32) << 16) + half * COLS;
#pragma unroll 1
  for (int c = 0; c < COLS; c += 8) {
    float v[8];
    ptx::tmem_ld8(taddr + c, v);
    if (row < S) run_prog<CHUNK>(P, G, (int64_t)b * S + row, half * COLS + c, 8, v, red);
  }
  ptx::tc_fence_before();
  if (row < S) {
    flush_reds(P, G, (int64_t)b * S + row, red);
  }
}

__device__ __noinline__ void run_attn(const Params& P, const Stage& st, char* smem) {
  SmemCtrl* ctl = ctrl_of(smem);
  TcState ts = ctl->ts;
  const Prog G = cached_prog(smem, 0);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, tid = threadIdx.x;
  char* base = smem + kCtrlBytes;
  char* Qs = base;               // [128 q][d] K-major, d/64 atoms of 16 KB
  char* Ks = base + 32768;       // [128 keys][d]
  char* Vt = base + 65536;       // [d][128 keys], 2 atoms of d*128 B
  char* Ps = base + 98304;       // [128 q][128 keys], 2 atoms of 16 KB
  const int S = st.at_S, d = st.at_d;
  const Addr& AQ = P.addrs[st.at_q];
  const Addr& AK = P.addrs[st.at_k];
  const Addr& AV = P.addrs[st.at_v];
  const uint16_t* gq = (const uint16_t*)addr_ptr(P, AQ) + AQ.base;
  const uint16_t* gk = (const uint16_t*)addr_ptr(P, AK) + AK.base;
  const uint16_t* gv = (const uint16_t*)addr_ptr(P, AV) + AV.base;
  float red[MAX_RED] = {0.f, 0.f, 0.f, 0.f};
  const float scale = st.at_scale;
  for (int b = blockIdx.x; b < st.at_B; b += gridDim.x) {
    if (tid == 0) mark(P, ctl, 0);
    const int64_t hb = (int64_t)b * S * d;
    // ---- stage Q, K (K-major, swizzled; head dim zero-padded to dk = 64 / 128 so every row is whole
    // 128-byte swizzle atoms) and V^T
    const int dk = (d + 63) & ~63;
    const int chunks = 128 * (dk / 8);
    for (int e = tid; e < chunks; e += kThreads) {
      int s = e / (dk / 8), c8 = e % (dk / 8);
      int atom = c8 / 8, cb = (c8 % 8) * 16;
      uint4 qv = make_uint4(0, 0, 0, 0), kv = make_uint4(0, 0, 0, 0), vv = make_uint4(0, 0, 0, 0);
      if (s < S && c8 * 8 < d) {
        qv = __ldcg(reinterpret_cast<const uint4*>(gq + hb + (int64_t)s * d + c8 * 8));
        kv = __ldcg(reinterpret_cast<const uint4*>(gk + hb + (int64_t)s * d + c8 * 8));
        vv = __ldcg(reinterpret_cast<const uint4*>(gv + hb + (int64_t)s * d + c8 * 8));
      }
      *reinterpret_cast<uint4*>(Qs + atom * 16384 + sw128(s, cb)) = qv;
      *reinterpret_cast<uint4*>(Ks + atom * 16384 + sw128(s, cb)) = kv;
      if (c8 * 8 < d) {
        const uint16_t* vp = reinterpret_cast<const uint16_t*>(&vv);
        int katom = s / 64, kb = (s % 64) * 2;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          int dd = c8 * 8 + j;
          *reinterpret_cast<uint16_t*>(Vt + katom * (d * 128) + sw128(dd, kb)) = vp[j];
        }
      }
    }
    ptx::fence_proxy_async();
    __syncthreads();
    if (tid == 0) mark(P, ctl, 1);   // Q, K, V^T staged
    // ---- S = Q K^T  (M=128 queries, N=128 keys, K=d) -> TMEM cols [0,128)
    if (warp == 1 && lane == 0) {
      ptx::tc_fence_after();
      const uint32_t idesc = ptx::idesc_bf16(128, 128);
      const uint32_t q0 = ptx::smem_u32(Qs), k0 = ptx::smem_u32(Ks);
      for (int ks = 0; ks < dk / 16; ++ks) {
        uint32_t off = (ks / 4) * 16384 + (ks % 4) * 32;
        ptx::mma_bf16(ctl->tmem_base, ptx::sdesc_sw128(q0 + off), ptx::sdesc_sw128(k0 + off), idesc, ks > 0);
      }
      ptx::mma_commit(&ctl->attb);
    }
    __syncwarp();
    // ---- softmax: warp w owns rows 32*(w%4).., the two warps of a row group split the keys
    {
      const int q = warp & 3, half = warp >> 2;
      const int row = q * 32 + lane;
      ptx::mbar_wait_wd(&ctl->attb, ts.att_phase);
      ptx::tc_fence_after();
      if (tid == 0) mark(P, ctl, 2);   // S ready
      // three cheap passes over TMEM (16 columns at a time) keep the register footprint small
      const uint32_t tb = ctl->tmem_base + ((uint32_t)(q * 32) << 16) + half * 64;
      float mx = -INFINITY;
      // additive score terms (e.g. relative-position bias, shifted-window mask): applied once, the
      // scaled + biased scores are written back to TMEM and the later passes use scale 1
      const bool adds = st.at_add[0] >= 0;
      const int nadd = adds ? (st.at_add[1] >= 0 ? 2 : 1) : 0;
      Addr AD[2];
      if (adds) AD[0] = P.addrs[st.at_add[0]];
      if (nadd > 1) AD[1] = P.addrs[st.at_add[1]];
      const float sc1 = adds ? 1.f : scale;
#pragma unroll 1
      for (int c0 = 0; c0 < 64; c0 += 16) {
        if (half * 64 + c0 >= S) break;
        float v[16];
        ptx::tmem_ld16(tb + c0, v);
        if (adds) {
          const int64_t r = (int64_t)b * S + row;
          float t[2][16];
#pragma unroll
          for (int k = 0; k < 2; ++k) {
#pragma unroll
            for (int j = 0; j < 16; ++j) t[k][j] = 0.f;
            if (k < nadd && row < S) {
              // every load of the 16 columns is issued before any is used
              const Addr& A = AD[k];
              const int64_t rb = A.mode == 0 ? A.base + r * A.rs : A.mode == 1 ? A.base + P.tabs[A.rtab + r] : 0;
#pragma unroll
              for (int j = 0; j < 16; ++j) {
                const int col = half * 64 + c0 + j;
                if (col < S) {
                  const int64_t o = A.mode == 0 ? rb + col * A.cs
                                  : A.mode == 1 ? rb + P.tabs[A.ctab + col] : addr_off(P, A, r, col);
                  t[k][j] = ld1(P, A, o);
                }
              }
            }
          }
#pragma unroll
          for (int j = 0; j < 16; ++j) v[j] = v[j] * scale + t[0][j] + t[1][j];
          ptx::tmem_st16(tb + c0, v);
        }
#pragma unroll
        for (int j = 0; j < 16; ++j)
          if (half * 64 + c0 + j < S) mx = fmaxf(mx, v[j] * sc1);
      }
      float* xch = reinterpret_cast<float*>(Qs);    // [2][128] exchange (Q is consumed by now)
      xch[half * 128 + row] = mx;
      __syncthreads();
      mx = fmaxf(mx, xch[(half ^ 1) * 128 + row]);
      float z = 0.f;
#pragma unroll 1
      for (int c0 = 0; c0 < 64; c0 += 16) {
        float v[16];
        ptx::tmem_ld16(tb + c0, v);
#pragma unroll
        for (int j = 0; j < 16; ++j)   // ex2.approx (rel. err ~2^-22): P is rounded to bf16 anyway
          if (half * 64 + c0 + j < S) z += __expf(v[j] * sc1 - mx);
      }
      __syncthreads();
      xch[half * 128 + row] = z;
      __syncthreads();
      z += xch[(half ^ 1) * 128 + row];
      const float iz = 1.f / z;
#pragma unroll 1
      for (int c0 = 0; c0 < 64; c0 += 16) {
        float v[16];
        ptx::tmem_ld16(tb + c0, v);
#pragma unroll
        for (int j = 0; j < 16; ++j) v[j] = (half * 64 + c0 + j < S) ? __expf(v[j] * sc1 - mx) * iz : 0.f;
#pragma unroll
        for (int h8 = 0; h8 < 16; h8 += 8) {
          uint32_t pk[4];
#pragma unroll
          for (int j = 0; j < 8; j += 2)
            pk[j / 2] = (uint32_t)f2bf(v[h8 + j]) | ((uint32_t)f2bf(v[h8 + j + 1]) << 16);
          *reinterpret_cast<uint4*>(Ps + half * 16384 + sw128(row, (c0 + h8) * 2)) =
              make_uint4(pk[0], pk[1], pk[2], pk[3]);
        }
      }
      ptx::tc_fence_before();
    }
    ts.att_phase ^= 1;
    ptx::fence_proxy_async();
    __syncthreads();
    if (tid == 0) mark(P, ctl, 3);   // softmax done, P staged
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
    ptx::mbar_wait_wd(&ctl->attb, ts.att_phase);
    ptx::tc_fence_after();
    if (tid == 0) mark(P, ctl, 4);   // O ready
    attn_epilogue(P, G, ctl, b, S, d, red);
    ts.att_phase ^= 1;
    __syncthreads();
    if (tid == 0) mark(P, ctl, 5);   // epilogue done
  }
  if (threadIdx.x == 0) ctl->ts = ts;
  __syncthreads();
}

// ================================================================== the persistent kernel
__global__ void __launch_bounds__(kThreads, 1) souffle_exec_kernel(const __grid_constant__ Params P) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  SmemCtrl* ctl = ctrl_of(smem);
  Stage* sst = stage_of(smem);
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) ctl->ts = TcState{0u, 0u, 0u, 0u};
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
  prefetch_stage(P, P.first, smem);   // the first stage never starts with a barrier
  for (int s = P.first; s < P.first + P.count; ++s) {
    if (threadIdx.x == 0) {
      ctl->cur_stage = s;
      if (P.prof && blockIdx.x == 0) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        P.prof[s] = t;
        P.prof[P.n_stages_total + 1 + 8 * s + 6] = (unsigned long long)clock64();   // SM clock at start
      }
    }
    progress(P, s, 0);
    __syncthreads();
    const Stage& st = *sst;
    // read before the stage's closing __syncthreads: once a thread is past it, prefetch_stage may
    // overwrite the staged descriptor with stage s+1's, and a lagging warp would then take s+1's
    // barrier decision (a mismatched barrier sequence that stalled one CTA forever)
    const bool bar = P.cooperative && st.barrier_after;
    switch (st.kind) {
      case ST_EW: run_ew(P, st, smem); break;
      case ST_REDUCE: run_reduce(P, st, smem); break;
      case ST_GEMM_SIMT: run_gemm_simt(P, st, smem); break;
      case ST_GEMM_TC: run_gemm_tc(P, st, smem); break;
      case ST_ATTN: run_attn(P, st, smem); break;
    }
    __syncthreads();
    if (s + 1 < P.first + P.count) {
      // split-phase barrier: arrive, prefetch the next stage's static data, then wait
      progress(P, s, 9);
      if (bar) barrier_arrive(P, nb, ctl);
      prefetch_stage(P, s + 1, smem);
      if (bar) barrier_wait(P, nb);
    }
  }
  // ---- exit: the last CTA resets the barrier words and clears the fused-reduction targets
  if (threadIdx.x == 0) {
    __threadfence();
    unsigned old = atomicAdd(&P.ctrl[1], 1u);
    ctl->flag = (old == gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  if (ctl->flag) {
    __threadfence();
    if (P.prof && threadIdx.x == 0) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      P.prof[P.first + P.count] = t;   // end of the launch (last CTA out)
    }
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
  // smem = the launch's working area (EXEC_SMEM) + its tensor-cache units; +1024 for the alignment
  constexpr int kMaxDyn = EXEC_SMEM + 1024 + EXEC_CACHE_FLOATS * 4;
  static_assert(kMaxDyn <= 227 * 1024, "exceeds the opt-in shared memory per block");
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(souffle_exec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxDyn);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = (smem > EXEC_SMEM ? smem : EXEC_SMEM) + 1024;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = cooperative ? 1 : 0;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, souffle_exec_kernel, prm);
}

cudaError_t exec_max_active(int smem, int* blocks) {
  constexpr int kMaxDyn = EXEC_SMEM + 1024 + EXEC_CACHE_FLOATS * 4;
  cudaError_t e = cudaFuncSetAttribute(souffle_exec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxDyn);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, souffle_exec_kernel, kThreads,
                                                       (smem > EXEC_SMEM ? smem : EXEC_SMEM) + 1024);
}

}  // namespace souffle
