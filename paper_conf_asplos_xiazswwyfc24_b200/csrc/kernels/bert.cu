// Specialised Souffle subprogram kernel for BERT encoder stacks on sm_100a (B200).
//
// The partitioner puts a whole BERT stack into one subprogram (§5.4; Table 5: Souffle
// runs BERT with very few kernels) and the lowering recognises the encoder-layer TE pattern
// (host/bert.cpp).  This kernel runs that subprogram as ONE persistent cooperative launch
// (§6.4 "global sync", Fig. 2):
//
//   warp 8      weight producer: walks the stage list and TMA-loads, for every GEMM task this CTA
//               owns, its weight K-chunks into a BW_SLOTS x 16 KB shared-memory ring.  Weights are
//               constants, so it runs ahead across grid barriers and the HBM weight stream overlaps
//               the activation dependency chain (§6.5 cross-stage prefetch, Table 4 V4).
//   warps 0-7   stage executor:
//     GEMM      A (bf16 activations) streamed by TMA through a BA_SLOTS-slot ring; one thread issues
//               tcgen05.mma (M = 128 tokens, N = tile, K = 16) into TMEM; fused epilogues:
//               bias + bf16 + head-major / transposed stores (QKV: the reshape/permute index maps
//               of §6.2 folded into the store), bias + erf-GELU (FFN1), or fp32 split-K partials;
//               stored straight from registers (every thread owns >= 16 contiguous bytes of a
//               token row, or a 64-byte coalesced run of V^T), the bias loaded during the mainloop.
//     ATTN      per head: Q, K, V^T by TMA, S = QK^T in TMEM, softmax (max-subtracted, fp32
//               registers), P bf16 in smem, O = PV in TMEM, ctx stored bf16 (Fig. 1(c), §2.3).
//     ROW       one CTA per token row: sum of the split-K partials + bias + residual, LayerNorm
//               with (mean, M2) statistics merged pairwise (one block reduction), fp32
//               and bf16 outputs (two-phase reduction: partial results per block,
//               combined after the global sync).
//   A split-phase grid barrier (one arrival counter per barrier) separates dependent stages.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../bert_types.h"
#include "ptx.cuh"

namespace souffle {
namespace bert {

static_assert(sizeof(BStage) % 16 == 0, "BStage is copied with 16-byte vectors");
static_assert(2 * sizeof(BStage) <= 1024, "two BStage buffers are staged in the control block");

struct Ctrl {
  uint64_t wfull[BW_SLOTS];
  uint64_t wempty[BW_SLOTS];
  uint64_t afull[BA_SLOTS];
  uint64_t aempty[BA_SLOTS];
  uint64_t accb;
  uint64_t recvb;               // cluster-pair split-K: the partner's half tile has landed
  uint64_t attb;
  uint64_t qkvb;
  uint32_t tmem_base;
  volatile int cur_stage;       // debug (dbg_skip bit 12): the producer does not run ahead of the executor
  float red[2][8];
};
static_assert(sizeof(Ctrl) <= 1024, "control block");

__device__ __forceinline__ void csync() { asm volatile("bar.sync 1, 256;" ::: "memory"); }

__device__ __forceinline__ uint32_t sw128(int row, int kbyte) {
  return (uint32_t)(row * 128 + ((((kbyte >> 4) ^ (row & 7)) & 7) << 4) + (kbyte & 15));
}
__device__ __forceinline__ uint32_t pack_bf16(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);   // .x = a (low half)
  return *reinterpret_cast<uint32_t*>(&h);
}
__device__ __forceinline__ uint16_t bf16_bits(float a) {
  __nv_bfloat16 b = __float2bfloat16_rn(a);
  return *reinterpret_cast<uint16_t*>(&b);
}
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
// the same GELU on two values with packed fp32 arithmetic (FFMA2 / FMUL2 / FADD2: every lane's result
// is the IEEE-rounded scalar result, so the output is bit-identical to gelu_erf; half the issue slots)
__device__ __forceinline__ float2 gelu_erf2(float2 x) {
  const float2 u = __fmul2_rn(x, make_float2(0.70710678118654752f, 0.70710678118654752f));
  const float2 t = make_float2(fminf(fabsf(u.x), 3.92f), fminf(fabsf(u.y), 3.92f));
  auto cc = [](float c) { return make_float2(c, c); };
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
  const float2 hx = __fmul2_rn(x, cc(0.5f));
  return __fmul2_rn(hx, __fadd2_rn(cc(1.f), e));   // (0.5 x)(1 + e), rounded as in gelu_erf
}
template <class T>
__device__ __forceinline__ const void* ldgp(T* const* p) {
  return (const void*)__ldg(reinterpret_cast<const unsigned long long*>(p));
}

__device__ __forceinline__ void mark(const BertParams& P, int idx) {
  if (P.prof && blockIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    P.prof[idx] = t;
  }
}
// debug timeline: sub-stage mark k of stage st (recorded by the first CTA with work in the stage)
__device__ __forceinline__ void submark(const BertParams& P, const BStage& st, int k) {
  if (P.prof && blockIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    P.prof[P.nstages + 2 + 16 * st.idx + k] = t;
  }
}

// watchdog for the spin waits: a dependency that never resolves (a planner bug) aborts the launch with
// an error after ~2 s instead of hanging the GPU
__device__ __forceinline__ void spin_guard(uint32_t& n, unsigned long long& t0) {
  if ((++n & 1023u) == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t0 == 0) t0 = t;
    else if (t - t0 > 2000000000ull) __trap();
  }
}

// ------------------------------------------------------------------ grid barrier (split phase)
__device__ __forceinline__ void grid_arrive(const BertParams& P, int k, bool tma_consumed) {
  // generic-proxy writes of this stage -> TMA reads of later stages (split-K partials are read by
  // plain loads of the LayerNorm rows: no proxy fence for those stages).  The data is global: the
  // proxy fence is restricted to the global state space (timing study bit 1 << 20: full fence)
  if (tma_consumed && !(P.dbg_skip & (1 << 24))) {   // timing study bit 24: no producer-side proxy fence
    if (P.dbg_skip & (1 << 20)) ptx::fence_proxy_async();
    else ptx::fence_proxy_async_global();
  }
  csync();
  if (threadIdx.x == 0) {
    if (P.dbg_skip & (1 << 21)) {
      __threadfence();
      atomicAdd(&P.ctrl[k], 1u);
    } else {
      ptx::red_release_add(&P.ctrl[k], 1u);   // release: orders the CTA's writes (bar.sync above) first
    }
  }
}
__device__ __forceinline__ void grid_wait(const BertParams& P, int k, int target_arrivals, bool tma_reads) {
  if (threadIdx.x == 0) {
    const unsigned target = (unsigned)target_arrivals;
    uint32_t n = 0;
    unsigned long long t0 = 0;
    // acquire polling: relaxed polling + one fence.acq_rel measured 23 us slower over the 72 barriers
    while (ptx::ld_acquire(&P.ctrl[k]) < target) spin_guard(n, t0);
    if (tma_reads) ptx::fence_proxy_async_global();   // the stage reads other CTAs' data through TMA
  }
  csync();
}

// point-to-point dependency: the producer CTA publishes its epilogue stores (generic proxy -> the
// consumer's TMA reads) and bumps one flag; the consumer polls only the flag of the data it reads
__device__ __forceinline__ void flag_signal(const BertParams& P, const BStage& st, int n0) {
  if (P.dbg_skip & (1 << 25)) ptx::fence_proxy_async();   // timing study bit 25: round-2 fences
  else ptx::fence_proxy_async_global();                    // the consumer's TMA reads global data
  csync();
  if (threadIdx.x == 0) {
    // the release below is cumulative over the CTA's writes ordered before it by bar.sync: no
    // separate gpu-scope fence
    if (P.dbg_skip & (1 << 25)) __threadfence();
    unsigned* f = st.fout + 32 * ((n0 % st.fmod) / st.fdiv);
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(f), "r"(1u) : "memory");
  }
}
__device__ __forceinline__ void flag_wait(const BertParams& P, const BStage& st, int idx) {
  if (threadIdx.x == 0) {
    const unsigned* f = st.fin + 32 * idx;
    uint32_t n = 0;
    unsigned long long t0 = 0;
    while (ptx::ld_acquire(f) < (unsigned)st.fneed) spin_guard(n, t0);
    if (P.dbg_skip & (1 << 25)) ptx::fence_proxy_async();
    else ptx::fence_proxy_async_global();
  }
  csync();
}

// does this CTA have work in stage st?  (GEMM: one task per CTA; ATTN: heads on the last CTAs;
// ROW: rows on the first CTAs)
__device__ __forceinline__ bool has_work(const BertParams& P, const BStage& st) {
  const int b = blockIdx.x;
  if (st.kind == BS_GEMM || st.kind == BS_ATTN) return b < st.ntasks;
  return st.row_mode == 0 || b < P.S;   // stage 0 (convert + constant refresh) runs on every CTA
}

// K-chunk order of a task: rotated by the CTA index so that the CTAs of a stage, which all read
// the same activation tile, spread their concurrent A requests over all L2 slices instead of
// hammering the lines of one chunk together (the accumulation order changes; the sum does not)
__device__ __forceinline__ int rot_chunk(const BertParams& P, int i, int nk) {
  if (P.dbg_skip & 8192) return i;                                    // timing study: no rotation
  if (P.dbg_skip & 16384) return (i + (int)blockIdx.x / 16) % nk;     // timing study: groups of 16 CTAs
  return (i + (int)blockIdx.x) % nk;
}

// weight K-chunks per ring slot for an N tile of nt rows (16 KB / (nt * 128 B))
__device__ __forceinline__ int wgroup(int nt) { return max(1, BW_SLOT_BYTES / (nt * 128)); }

// ------------------------------------------------------------------ weight producer (warp 8)
__device__ void weight_producer(const BertParams& P, Ctrl* C, char* wring) {
  const char* tmaps = (const char*)P.tmaps;
  uint32_t it = 0;
  for (int s = P.s_begin; s < P.s_end; ++s) {
    const BStage* st = P.stages + s;
    const int kind = __ldg(&st->kind);
    if (kind != BS_GEMM && kind != BS_ATTN) continue;   // ATTN: fused out-projection tile
    if (P.dbg_skip & 4096)
      while (C->cur_stage < s) {
      }
    const int task = blockIdx.x;
    if (task >= __ldg(&st->ntasks)) continue;
    const int nsplit = __ldg(&st->nsplit), nt = __ldg(&st->nt), kch = __ldg(&st->kchunks);
    const int wrows = __ldg(&st->wrows), wmap0 = __ldg(&st->wmap0);
    const int tile = task / nsplit, split = task % nsplit;
    const int n0 = tile * nt;
    const int map = wmap0 + n0 / wrows, row = n0 % wrows;
    const int kc0 = split * kch;
    const int nk = min(kch, __ldg(&st->K) / 64 - kc0);
    const int gsz = wgroup(nt);
    for (int c0 = 0; c0 < nk; c0 += gsz, ++it) {
      const int cnt = min(gsz, nk - c0);
      const uint32_t slot = it % BW_SLOTS, ph = (it / BW_SLOTS) & 1;
      ptx::mbar_wait(&C->wempty[slot], ph ^ 1);
      ptx::mbar_arrive_expect_tx(&C->wfull[slot], (uint32_t)(cnt * nt * 128));
      for (int j = 0; j < cnt; ++j)
        ptx::tma_load_2d(wring + slot * BW_SLOT_BYTES + j * nt * 128, tmaps + 128 * map, &C->wfull[slot],
                         (kc0 + rot_chunk(P, c0 + j, nk)) * 64, row);
    }
  }
}

// ------------------------------------------------------------------ GEMM stage
struct MmaState {
  uint32_t wit;            // weight-ring consumer group counter (thread 0)
  uint32_t aload, ause;    // A-ring chunk counters (thread 0)
  uint32_t accph, attph, qkvph, recvph;
};

// Epilogue of one 128 x nt accumulator tile, straight from registers: warp w reads TMEM lanes
// 32*(w%4).. (token rows) and column half w/4, adds the bias it loaded while the MMAs ran
// (bias_half: COLS fp32 values of this thread's half, 16-byte aligned), and stores its row segment:
// fp32 partial (COLS*4 B), bf16 GELU / Q / K (COLS*2 B >= 16 B) or V^T (one bf16 per feature row;
// the 32 lanes of a warp write 64 contiguous bytes).  Rows >= S (TMA zero-fill) are not stored.
template <int COLS>
__device__ __forceinline__ void tmem_row(Ctrl* C, float* v) {
  const int warp = threadIdx.x >> 5;
  const uint32_t taddr = C->tmem_base + ((uint32_t)((warp & 3) * 32) << 16) + (warp >> 2) * COLS;
  if constexpr (COLS == 8) ptx::tmem_ld8(taddr, v);
  else if constexpr (COLS == 16) ptx::tmem_ld16(taddr, v);
  else if constexpr (COLS == 32) ptx::tmem_ld32(taddr, v);
  else ptx::tmem_ld64(taddr, v);
  ptx::tc_fence_before();
}

// fp32 split-K partial [split][S][N] (out-projection per head, FFN2 per K range): no bias.  Staged
// through shared memory (the A region: its MMAs have completed) so every warp store instruction
// writes 512 contiguous bytes -- thread-per-row float4 stores touch 32 lines per instruction and
// measured 2x slower for these 32 KB tiles.  mk: debug mark index.
template <int COLS>
__device__ __forceinline__ void tail_partial(const BertParams& P, const BStage& st, Ctrl* C, MmaState& ms, int n0,
                                             int split, char* stage_smem, int mk) {
  ptx::mbar_wait(&C->accb, ms.accph);
  ms.accph ^= 1;
  ptx::tc_fence_after();
  if (threadIdx.x == 0) submark(P, st, mk);
  float v[COLS];
  tmem_row<COLS>(C, v);
  const int tid = threadIdx.x, warp = tid >> 5, half = warp >> 2, row = (warp & 3) * 32 + (tid & 31);
  constexpr int NT = 2 * COLS, LD = NT + 4;   // padded fp32 row stride of the staging tile
  float* stg = reinterpret_cast<float*>(stage_smem);
#pragma unroll
  for (int c = 0; c < COLS; c += 4)
    *reinterpret_cast<float4*>(stg + row * LD + half * COLS + c) = make_float4(v[c], v[c + 1], v[c + 2], v[c + 3]);
  csync();
  constexpr int U = NT / 4;   // float4 units per row
  const int S = P.S, N = st.N;
  float* dst = st.part + (int64_t)split * S * N + n0;
  for (int u = tid; u < S * U; u += BERT_COMPUTE) {
    const int r = u / U, c4 = u % U;
    *reinterpret_cast<float4*>(dst + (int64_t)r * N + 4 * c4) = *reinterpret_cast<const float4*>(stg + r * LD + 4 * c4);
  }
  // the staging tile is generic-proxy data in the region the next stage's TMA writes: every writer
  // orders its shared-memory stores before those async-proxy writes (CTA-local proxy fence)
  ptx::fence_proxy_async_smem();
}

// + bias, then erf-GELU -> bf16 [S][N] (FFN1), or bf16 Q / K head-major and V^T (QKV, the reshape /
// permute index maps of §6.2 folded into the store).  Tiles of <= 32 columns load their bias while
// the MMAs run (warps 2-7 are idle in the mainloop); wider tiles after the accumulator.
template <int COLS>
__device__ __forceinline__ void tail_bias(const BertParams& P, const BStage& st, Ctrl* C, MmaState& ms, int n0) {
  const int warp = threadIdx.x >> 5, half = warp >> 2, row = (warp & 3) * 32 + (threadIdx.x & 31);
  const int c0 = n0 + half * COLS;
  constexpr bool kEarly = COLS <= 16;
  float4 bq[kEarly ? COLS / 4 : 1];
  if constexpr (kEarly) {
#pragma unroll
    for (int c = 0; c < COLS; c += 4) bq[c / 4] = __ldg(reinterpret_cast<const float4*>(st.bias + c0 + c));
  }
  ptx::mbar_wait(&C->accb, ms.accph);
  ms.accph ^= 1;
  ptx::tc_fence_after();
  if (threadIdx.x == 0) submark(P, st, 3);
  float v[COLS];
  tmem_row<COLS>(C, v);
  if (row >= P.S) return;
#pragma unroll
  for (int c = 0; c < COLS; c += 4) {
    const float4 b = kEarly ? bq[kEarly ? c / 4 : 0] : __ldg(reinterpret_cast<const float4*>(st.bias + c0 + c));
    v[c] += b.x; v[c + 1] += b.y; v[c + 2] += b.z; v[c + 3] += b.w;
  }
  const int S = P.S, N = st.N;
  if (st.epi == EP_GELU) {
#pragma unroll
    for (int c = 0; c < COLS; ++c) v[c] = gelu_erf(v[c]);
    uint4* dst = reinterpret_cast<uint4*>(st.out_b + (int64_t)row * N + c0);
#pragma unroll
    for (int c = 0; c < COLS; c += 8)
      dst[c / 8] = make_uint4(pack_bf16(v[c], v[c + 1]), pack_bf16(v[c + 2], v[c + 3]), pack_bf16(v[c + 4], v[c + 5]),
                              pack_bf16(v[c + 6], v[c + 7]));
    return;
  }
  // EP_QKV: columns [n0, n0 + 2*COLS) of [Q | K | V] lie in one head (the tile width divides 64)
  const int H = N / 3;
  const int which = n0 / H, hh = (n0 % H) >> 6, jd = (n0 & 63) + half * COLS;
  if (which < 2) {   // head-major [S][64]: COLS*2 contiguous bytes per token row
    uint4* dst = reinterpret_cast<uint4*>(st.out_b + (((int64_t)(which * st.heads + hh) * S + row) << 6) + jd);
#pragma unroll
    for (int c = 0; c < COLS; c += 8)
      dst[c / 8] = make_uint4(pack_bf16(v[c], v[c + 1]), pack_bf16(v[c + 2], v[c + 3]), pack_bf16(v[c + 4], v[c + 5]),
                              pack_bf16(v[c + 6], v[c + 7]));
  } else {           // V^T [64][S]: a warp writes 32 consecutive tokens (64 B) of one feature row
    uint16_t* dst = st.out_vt + ((int64_t)hh * 64 + jd) * S + row;
#pragma unroll
    for (int c = 0; c < COLS; ++c) dst[(int64_t)c * S] = bf16_bits(v[c]);
  }
}

// Cluster-pair split-K (st.cpair): the two CTAs of a cluster computed the two K halves of the same
// 128 x (4 HC) tile.  CTA rank r finalises columns [2 HC r, 2 HC r + 2 HC): it sends the partner's
// columns of its partial into the partner's shared memory (one DSMEM bulk copy), then
// adds the partner's contribution to its own half and runs the fused epilogue on HC columns per warp
// half.  The A bytes each CTA streams are halved (K / 2) for one 8-16 KB exchange.
template <int HC>
__device__ __forceinline__ void pair_tail(const BertParams& P, const BStage& st, Ctrl* C, MmaState& ms, int n0,
                                          char* recv, char* stage) {
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int q = warp & 3, half = warp >> 2, row = q * 32 + lane;
  const uint32_t rank = (uint32_t)blockIdx.x & 1u;   // == split == cluster rank
  const int c0 = n0 + (int)rank * 2 * HC + half * HC;
  float4 bq[HC / 4];
#pragma unroll
  for (int c = 0; c < HC; c += 4) bq[c / 4] = __ldg(reinterpret_cast<const float4*>(st.bias + c0 + c));
  ptx::mbar_wait(&C->accb, ms.accph);
  ms.accph ^= 1;
  ptx::tc_fence_after();
  if (tid == 0) submark(P, st, 3);
  const uint32_t lanes = C->tmem_base + ((uint32_t)(q * 32) << 16);
  constexpr uint32_t kBytes = 128 * 2 * HC * 4;
  if (tid == 0) ptx::mbar_arrive_expect_tx(&C->recvb, kBytes);   // the partner's half tile, by bulk copy
  float v[HC];
  // ---- the partner's columns of this partial -> local staging (the A ring: its MMAs completed), then
  // one bulk DSMEM copy into the partner's receive buffer, completing on the partner's mbarrier
  if constexpr (HC == 8) ptx::tmem_ld8(lanes + (rank ^ 1u) * 2 * HC + half * HC, v);
  else ptx::tmem_ld16(lanes + (rank ^ 1u) * 2 * HC + half * HC, v);
  // the exchanged half tile is [128 rows][2 HC] fp32 with its 16-byte chunks XOR-swizzled by row (the
  // lanes of a warp are consecutive rows: unswizzled, every lane would hit the same banks)
  constexpr int CPR = HC / 2;   // 16-byte chunks per row
  const int swz = (row * CPR >> 3) & (CPR - 1);
  float* stg = reinterpret_cast<float*>(stage) + row * 2 * HC;
#pragma unroll
  for (int c = 0; c < HC; c += 4)
    *reinterpret_cast<float4*>(stg + 4 * (((half * HC + c) >> 2) ^ swz)) = make_float4(v[c], v[c + 1], v[c + 2], v[c + 3]);
  // ---- own columns
  if constexpr (HC == 8) ptx::tmem_ld8(lanes + rank * 2 * HC + half * HC, v);
  else ptx::tmem_ld16(lanes + rank * 2 * HC + half * HC, v);
  ptx::tc_fence_before();
  ptx::fence_proxy_async_smem();   // generic smem writes -> the async-proxy bulk copy
  csync();
  if (tid == 0)
    ptx::bulk_s2cluster(ptx::mapa(ptx::smem_u32(recv), rank ^ 1u), stage, kBytes,
                        ptx::mapa(ptx::smem_u32(&C->recvb), rank ^ 1u));
  // the staging area is next written by a TMA load of a later stage, which comes after a grid
  // barrier that the partner only reaches once this copy has completed on its mbarrier
  ptx::mbar_wait(&C->recvb, ms.recvph);
  ms.recvph ^= 1;
  if (tid == 0) submark(P, st, 8);
  if (row >= P.S) return;
  const float* rp = reinterpret_cast<const float*>(recv) + row * 2 * HC;
#pragma unroll
  for (int c = 0; c < HC; c += 4) {
    const float4 o = *reinterpret_cast<const float4*>(rp + 4 * (((half * HC + c) >> 2) ^ swz));
    const float4 b = bq[c / 4];
    v[c] += o.x + b.x; v[c + 1] += o.y + b.y; v[c + 2] += o.z + b.z; v[c + 3] += o.w + b.w;
  }
  const int S = P.S, N = st.N;
  if (tid == 0) submark(P, st, 9);
  if (st.epi == EP_GELU) {
    if (!(P.dbg_skip & (1 << 22))) {   // timing study bit 22: no GELU (wrong values)
#pragma unroll
      for (int c = 0; c < HC; c += 2) {
        const float2 gg = gelu_erf2(make_float2(v[c], v[c + 1]));
        v[c] = gg.x;
        v[c + 1] = gg.y;
      }
    }
    if (tid == 0) submark(P, st, 10);
    if constexpr (HC == 16) {   // the row's 16 outputs = one 32-byte sector: one 256-bit store
      uint32_t u[8];
#pragma unroll
      for (int c = 0; c < 8; ++c) u[c] = pack_bf16(v[2 * c], v[2 * c + 1]);
      asm volatile("st.global.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(st.out_b + (int64_t)row * N + c0),
                   "r"(u[0]), "r"(u[1]), "r"(u[2]), "r"(u[3]), "r"(u[4]), "r"(u[5]), "r"(u[6]), "r"(u[7])
                   : "memory");
    } else {
      uint4* dst = reinterpret_cast<uint4*>(st.out_b + (int64_t)row * N + c0);
#pragma unroll
      for (int c = 0; c < HC; c += 8)
        dst[c / 8] = make_uint4(pack_bf16(v[c], v[c + 1]), pack_bf16(v[c + 2], v[c + 3]), pack_bf16(v[c + 4], v[c + 5]),
                                pack_bf16(v[c + 6], v[c + 7]));
    }
    if (tid == 0) submark(P, st, 11);
    return;
  }
  const int H = N / 3;   // EP_QKV (HC columns inside one head)
  const int which = c0 / H, hh = (c0 % H) >> 6, jd = c0 & 63;
  if (which < 2) {
    uint4* dst = reinterpret_cast<uint4*>(st.out_b + (((int64_t)(which * st.heads + hh) * S + row) << 6) + jd);
#pragma unroll
    for (int c = 0; c < HC; c += 8)
      dst[c / 8] = make_uint4(pack_bf16(v[c], v[c + 1]), pack_bf16(v[c + 2], v[c + 3]), pack_bf16(v[c + 4], v[c + 5]),
                              pack_bf16(v[c + 6], v[c + 7]));
  } else {
    uint16_t* dst = st.out_vt + ((int64_t)hh * 64 + jd) * S + row;
#pragma unroll
    for (int c = 0; c < HC; ++c) dst[(int64_t)c * S] = bf16_bits(v[c]);
  }
}

template <int COLS>
__device__ __forceinline__ void gemm_tail(const BertParams& P, const BStage& st, Ctrl* C, MmaState& ms, int n0,
                                          int split, char* areg) {
  if (st.epi == EP_PARTIAL) tail_partial<COLS>(P, st, C, ms, n0, split, areg, 3);
  else tail_bias<COLS>(P, st, C, ms, n0);
}

__device__ void run_gemm(const BertParams& P, const BStage& st, Ctrl* C, char* wring, char* areg, MmaState& ms) {
  const int task = blockIdx.x;
  if (task >= st.ntasks) return;
  const int tid = threadIdx.x, warp = tid >> 5;
  const int tile = task / st.nsplit, split = task % st.nsplit;
  const int nt = st.nt, n0 = tile * nt;
  const int kc0 = split * st.kchunks;
  const int nk = min(st.kchunks, st.K / 64 - kc0);
  const char* amap = (const char*)P.tmaps + 128 * st.amap;

  if (warp == 1) {
    // ---- A producer (warp 1, one elected lane issues): keeps BA_SLOTS chunks in flight, refills a
    // slot as soon as the MMAs that read it have completed
    for (int c = 0; c < nk; ++c) {
      const uint32_t slot = ms.aload % BA_SLOTS;
      if (ms.aload >= BA_SLOTS) ptx::mbar_wait(&C->aempty[slot], ((ms.aload / BA_SLOTS) - 1) & 1);
      if (ptx::elect_one()) {
        ptx::mbar_arrive_expect_tx(&C->afull[slot], BA_SLOT_BYTES);
        ptx::tma_load_2d(areg + slot * BA_SLOT_BYTES, amap, &C->afull[slot], (kc0 + rot_chunk(P, c, nk)) * 64, 0);
      }
      __syncwarp();
      ++ms.aload;
    }
  } else if (warp == 0) {
    // ---- MMA issue: the whole warp runs the loop (operands stay warp-uniform), one lane issues
    if (tid == 0) submark(P, st, 0);
    const uint32_t idesc = ptx::idesc_bf16(128, nt);
    const int gsz = wgroup(nt);
    const uint32_t tmem = C->tmem_base;
    const uint64_t da0 = ptx::sdesc_sw128(ptx::smem_u32(areg)), db0 = ptx::sdesc_sw128(ptx::smem_u32(wring));
    uint32_t wslot = 0;
    for (int c = 0; c < nk; ++c) {
      const uint32_t as = ms.ause % BA_SLOTS;
      ptx::mbar_wait(&C->afull[as], (ms.ause / BA_SLOTS) & 1);
      const int j = c % gsz;
      if (j == 0) {
        wslot = ms.wit % BW_SLOTS;
        ptx::mbar_wait(&C->wfull[wslot], (ms.wit / BW_SLOTS) & 1);
      }
      if (c == 0) {
        if (tid == 0) submark(P, st, 1);
        ptx::tc_fence_after();
      }
      const uint64_t da = da0 + (uint64_t)((as * BA_SLOT_BYTES) >> 4);
      const uint64_t db = db0 + (uint64_t)((wslot * BW_SLOT_BYTES + j * nt * 128) >> 4);
      const bool last_in_group = (j == gsz - 1 || c == nk - 1);
      if (ptx::elect_one()) {
        ptx::mma_bf16_k64(tmem, da, db, idesc, c > 0 ? 1u : 0u);
        ptx::mma_commit(&C->aempty[as]);
        if (last_in_group) ptx::mma_commit(&C->wempty[wslot]);
        if (c == nk - 1) ptx::mma_commit(&C->accb);
      }
      __syncwarp();
      ++ms.ause;
      if (last_in_group) ++ms.wit;
    }
    if (tid == 0) submark(P, st, 2);    // all MMAs issued
  }

  // ---- epilogue (all 8 warps: warp w reads TMEM lanes 32*(w%4).., column half w/4)
  if (st.cpair) {
    char* recv = areg + B_AREGION;
    if (nt == 32) pair_tail<8>(P, st, C, ms, n0, recv, areg);
    else pair_tail<16>(P, st, C, ms, n0, recv, areg);
    if (tid == 0) submark(P, st, 4);
    return;
  }
  switch (nt) {
    case 16: gemm_tail<8>(P, st, C, ms, n0, split, areg); break;
    case 32: gemm_tail<16>(P, st, C, ms, n0, split, areg); break;
    case 64: gemm_tail<32>(P, st, C, ms, n0, split, areg); break;
    default: gemm_tail<64>(P, st, C, ms, n0, split, areg); break;
  }
  if (tid == 0) submark(P, st, 4);
  if (st.fout) flag_signal(P, st, n0);
}

// ------------------------------------------------------------------ attention stage
// Attention of head h fused with its slice of the output projection (§6.1 horizontal + §6.2
// vertical: ctx_h never leaves the SM).  out = ctx Wo^T = sum_h ctx_h Wo[:, h-slice]^T, so CTA
// (tile j, head h) computes softmax(Q_h K_h^T / sqrt(d)) V_h and multiplies it by the Wo tile
// [rows j*nt.., cols h*64..] (one 64-wide K chunk, streamed by the weight producer); the result is
// head h's split-K partial of the out-projection, summed by the LayerNorm row stage.  Every
// N tile recomputes the (cheap) attention of its head instead of waiting for a grid barrier.
__device__ void run_attn(const BertParams& P, const BStage& st, Ctrl* C, char* wring, char* areg, MmaState& ms) {
  const int task = blockIdx.x;   // (see the weight producer: task = N tile * heads + head)
  if (task >= st.ntasks) return;
  const int h = task % st.heads, jt = task / st.heads;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int S = P.S;
  char* Qs = areg;                // [128 q][64 d]  one 16 KB atom; later the bf16 ctx_h tile (A operand)
  char* Ks = areg + 16384;        // [128 keys][64 d]
  char* Vt = areg + 32768;        // [64 d][128 keys]: 2 atoms of 8 KB (64 keys each)
  char* Ps = areg + 49152;        // [128 q][128 keys]: 2 atoms of 16 KB
  const char* tmaps = (const char*)P.tmaps;
  const uint32_t tmem = C->tmem_base;
  if (tid == 0) {
    ptx::mbar_arrive_expect_tx(&C->qkvb, 3 * 16384);
    ptx::tma_load_3d(Qs, tmaps + 128 * st.qkmap, &C->qkvb, 0, 0, h);
    ptx::tma_load_3d(Ks, tmaps + 128 * st.qkmap, &C->qkvb, 0, 0, st.heads + h);
    ptx::tma_load_3d(Vt, tmaps + 128 * st.vtmap, &C->qkvb, 0, 0, h);
    ptx::tma_load_3d(Vt + 8192, tmaps + 128 * st.vtmap, &C->qkvb, 64, 0, h);
    submark(P, st, 0);
  }
  ptx::mbar_wait(&C->qkvb, ms.qkvph);
  ms.qkvph ^= 1;
  if (tid == 0) submark(P, st, 1);
  // ---- S = Q K^T  (M = 128 queries, N = 128 keys, K = 64) -> TMEM columns [0, 128)
  if (warp == 0) {
    ptx::tc_fence_after();
    const uint32_t idesc = ptx::idesc_bf16(128, 128);
    const uint64_t dq = ptx::sdesc_sw128(ptx::smem_u32(Qs)), dk = ptx::sdesc_sw128(ptx::smem_u32(Ks));
    if (ptx::elect_one()) {
      ptx::mma_bf16_k64(tmem, dq, dk, idesc, 0u);
      ptx::mma_commit(&C->attb);
    }
    __syncwarp();
  }
  const int q = warp & 3, half = warp >> 2;
  const int row = q * 32 + lane;
  // ---- softmax: warp w owns TMEM lanes 32*(w%4).., the two warps of a lane group split the keys
  {
    ptx::mbar_wait(&C->attb, ms.attph);
    ms.attph ^= 1;
    ptx::tc_fence_after();
    if (tid == 0) submark(P, st, 2);
    const uint32_t tb = tmem + ((uint32_t)(q * 32) << 16) + half * 64;
    // p_j = 2^(s_j c - m c) / z with c = scale * log2(e): one FFMA + one MUFU.EX2 per score
    const float c = st.scale * 1.4426950408889634f;
    float sv[64];
    ptx::tmem_ld64(tb, sv);
    if (S < 128) {   // keys beyond S (TMA zero-fill)
#pragma unroll
      for (int j = 0; j < 64; ++j)
        if (half * 64 + j >= S) sv[j] = -INFINITY;
    }
    float m4[4] = {sv[0], sv[1], sv[2], sv[3]};   // 4 independent chains (no 64-long dependency)
#pragma unroll
    for (int j = 4; j < 64; ++j) m4[j & 3] = fmaxf(m4[j & 3], sv[j]);
    const float mx = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3]));
    // each half normalises with its own max; one (max, sum) exchange combines the halves:
    // z = z_a 2^{(m_a - m)c} + z_b 2^{(m_b - m)c}, p_j = 2^{(s_j - m_a)c} 2^{(m_a - m)c} / z
    const float mxs = (mx == -INFINITY) ? 0.f : mx;   // a fully masked half contributes 0
    const float mc = mxs * c;
    float z4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int j = 0; j < 64; ++j) {
      sv[j] = ptx::ex2(fmaf(sv[j], c, -mc));
      z4[j & 3] += sv[j];
    }
    const float z = (z4[0] + z4[1]) + (z4[2] + z4[3]);
    float2* xch = reinterpret_cast<float2*>(Qs);   // [2][128] (max, sum); Q is consumed (S complete)
    xch[half * 128 + row] = make_float2(mx, z);
    csync();
    const float2 o = xch[(half ^ 1) * 128 + row];
    const float m = fmaxf(mx, o.x);
    const float fa = ptx::ex2((mxs - m) * c);
    const float zt = z * fa + (o.x == -INFINITY ? 0.f : o.y * ptx::ex2((o.x - m) * c));
    const float iz = fa / zt;   // p_j = sv[j] * iz
#pragma unroll
    for (int c0 = 0; c0 < 64; c0 += 8) {
      *reinterpret_cast<uint4*>(Ps + half * 16384 + sw128(row, c0 * 2)) =
          make_uint4(pack_bf16(sv[c0] * iz, sv[c0 + 1] * iz), pack_bf16(sv[c0 + 2] * iz, sv[c0 + 3] * iz),
                     pack_bf16(sv[c0 + 4] * iz, sv[c0 + 5] * iz), pack_bf16(sv[c0 + 6] * iz, sv[c0 + 7] * iz));
    }
    ptx::tc_fence_before();
  }
  ptx::fence_proxy_async_smem();   // P / ctx smem writes -> the MMA (async proxy)
  csync();
  if (tid == 0) submark(P, st, 3);
  // ---- O = P V  (M = 128, N = 64, K = 128 keys) -> TMEM columns [128, 192)
  if (warp == 0) {
    ptx::tc_fence_after();
    const uint32_t idesc = ptx::idesc_bf16(128, 64);
    const uint64_t dp = ptx::sdesc_sw128(ptx::smem_u32(Ps)), dv = ptx::sdesc_sw128(ptx::smem_u32(Vt));
    if (ptx::elect_one()) {
      ptx::mma_bf16_k64(tmem + 128, dp, dv, idesc, 0u);
      ptx::mma_bf16_k64(tmem + 128, dp + 1024, dv + 512, idesc, 1u);
      ptx::mma_commit(&C->attb);
    }
    __syncwarp();
  }
  ptx::mbar_wait(&C->attb, ms.attph);
  ms.attph ^= 1;
  ptx::tc_fence_after();
  if (tid == 0) submark(P, st, 4);
  // ---- ctx_h (bf16) -> smem as the A operand [128 rows][64 K] of the out-projection tile
  {
    float o[32];
    ptx::tmem_ld32(tmem + 128 + ((uint32_t)(q * 32) << 16) + half * 32, o);
#pragma unroll
    for (int j = 0; j < 4; ++j)
      *reinterpret_cast<uint4*>(Qs + sw128(row, (half * 32 + 8 * j) * 2)) =
          make_uint4(pack_bf16(o[8 * j], o[8 * j + 1]), pack_bf16(o[8 * j + 2], o[8 * j + 3]),
                     pack_bf16(o[8 * j + 4], o[8 * j + 5]), pack_bf16(o[8 * j + 6], o[8 * j + 7]));
    ptx::tc_fence_before();
  }
  ptx::fence_proxy_async_smem();   // P / ctx smem writes -> the MMA (async proxy)
  csync();
  // ---- partial_h = ctx_h Wo[tile rows, h-slice]^T  (M = 128, N = nt, K = 64) -> TMEM columns [0, nt)
  if (warp == 0) {
    const uint32_t wslot = ms.wit % BW_SLOTS;
    ptx::mbar_wait(&C->wfull[wslot], (ms.wit / BW_SLOTS) & 1);
    ptx::tc_fence_after();
    const uint32_t idesc = ptx::idesc_bf16(128, st.nt);
    const uint64_t da = ptx::sdesc_sw128(ptx::smem_u32(Qs));
    const uint64_t db = ptx::sdesc_sw128(ptx::smem_u32(wring + wslot * BW_SLOT_BYTES));
    if (ptx::elect_one()) {
      ptx::mma_bf16_k64(tmem, da, db, idesc, 0u);
      ptx::mma_commit(&C->wempty[wslot]);
      ptx::mma_commit(&C->accb);
    }
    __syncwarp();
    ++ms.wit;
  }
  // split index = head, N tile = jt (EP_PARTIAL: no bias); staging in the consumed Q/K region
  switch (st.nt) {
    case 16: tail_partial<8>(P, st, C, ms, jt * st.nt, h, areg, 5); break;
    case 32: tail_partial<16>(P, st, C, ms, jt * st.nt, h, areg, 5); break;
    case 64: tail_partial<32>(P, st, C, ms, jt * st.nt, h, areg, 5); break;
    default: tail_partial<64>(P, st, C, ms, jt * st.nt, h, areg, 5); break;
  }
}

// ------------------------------------------------------------------ row stage (one CTA per row)
// Row statistics by pairwise (Chan) merging of (mean, M2 = sum of squared deviations): every
// thread centres its own 4 values exactly, equal-count merges in the warp tree, then the warps in
// order.  A constant row gives mean = the value and M2 = 0 exactly (so LayerNorm outputs beta, as
// the fp64 definition does), and an offset row (1e3 + noise) keeps the noise (no E[x^2] - E[x]^2
// cancellation).  Active threads = whole warps (cols is a multiple of 128); returns (mean, M2).
__device__ __forceinline__ float2 block_welford(Ctrl* C, float m, float M2, int nwarps) {
  float n = 4.f;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const float mb = __shfl_xor_sync(0xffffffffu, m, o);
    const float Mb = __shfl_xor_sync(0xffffffffu, M2, o);
    const float dl = mb - m;
    M2 = (M2 + Mb) + dl * dl * (0.5f * n);
    m = (m + mb) * 0.5f;   // commutative: both lanes of a pair hold the identical value
    n *= 2.f;
  }
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) == 0 && w < nwarps) {
    C->red[0][w] = m;
    C->red[1][w] = M2;
  }
  csync();
  // merge warp k (128 values) into warps 0..k-1 (128 k values): mean += dl / (k+1),
  // M2 += M2_k + dl^2 * 128 k / (k+1)
  float mean = C->red[0][0], q = C->red[1][0];
#pragma unroll
  for (int k = 1; k < 8; ++k) {
    if (k < nwarps) {
      const float dl = C->red[0][k] - mean;
      const float f = 1.f / (float)(k + 1);   // constant-folded
      mean += dl * f;
      q += C->red[1][k] + dl * dl * (128.f * (float)k * f);
    }
  }
  return make_float2(mean, q);
}

constexpr int kMaxSplit = 12;   // split-K partials summed by a LayerNorm row
// stage 0, all CTAs: refresh the packed constant vectors (bias / gamma / beta) from the bound
// pointers, so the later stages (which read the packed copy: a few 2 MB pages instead of ~200
// scattered allocations) always see the current parameter values
__device__ void refresh_consts(const BertParams& P) {
  for (int e = blockIdx.x; e < P.ncopies; e += gridDim.x) {   // one vector per CTA (n % 4 == 0)
    const BCopy* cp = P.copies + e;
    const float4* src = reinterpret_cast<const float4*>(ldgp(&cp->src));
    float4* dst = (float4*)__ldg(reinterpret_cast<const unsigned long long*>(&cp->dst));
    const int n4 = __ldg(&cp->n) >> 2;
    for (int k = threadIdx.x; k < n4; k += BERT_COMPUTE) dst[k] = __ldg(src + k);
  }
}

// one CTA per token row; thread t < cols/4 owns columns 4t..4t+3 (cols <= 1024)
__device__ void run_row(const BertParams& P, const BStage& st, Ctrl* C) {
  const int tid = threadIdx.x;
  const int S = P.S, cols = st.cols;
  const bool mine = 4 * tid < cols;
  for (int r = blockIdx.x; r < S; r += gridDim.x) {
    if (st.row_mode == 0) {
      if (mine) {
        const float4 x = __ldg(reinterpret_cast<const float4*>(st.r_in + (int64_t)r * cols) + tid);
        reinterpret_cast<uint2*>(st.r_out_b + (int64_t)r * cols)[tid] = make_uint2(pack_bf16(x.x, x.y), pack_bf16(x.z, x.w));
      }
      continue;
    }
    // sum of the split-K partials + bias + residual: every load of the row is issued before any is
    // used (one L2 round trip)
    const int ns = st.r_nsplit;
    const float* part = st.r_in + (int64_t)r * cols;
    const int64_t pstride = (int64_t)S * cols;
    float4 v = make_float4(0.f, 0.f, 0.f, 0.f), g = v, be = v;
    float m = 0.f, M2 = 0.f;
    if (mine) {
      const float4 b = __ldg(reinterpret_cast<const float4*>(st.r_bias) + tid);
      const float4 x = __ldcg(reinterpret_cast<const float4*>(st.r_res + (int64_t)r * cols) + tid);
      float4 t[kMaxSplit];
#pragma unroll
      for (int u = 0; u < kMaxSplit; ++u)
        t[u] = u < ns ? __ldcg(reinterpret_cast<const float4*>(part + u * pstride) + tid) : make_float4(0.f, 0.f, 0.f, 0.f);
      g = __ldg(reinterpret_cast<const float4*>(st.r_gamma) + tid);
      be = __ldg(reinterpret_cast<const float4*>(st.r_beta) + tid);
      float4 a = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int u = 0; u < kMaxSplit; ++u) { a.x += t[u].x; a.y += t[u].y; a.z += t[u].z; a.w += t[u].w; }
      v = make_float4((b.x + x.x) + a.x, (b.y + x.y) + a.y, (b.z + x.z) + a.z, (b.w + x.w) + a.w);
      m = ((v.x + v.y) + (v.z + v.w)) * 0.25f;
      const float d0 = v.x - m, d1 = v.y - m, d2 = v.z - m, d3 = v.w - m;
      M2 = (d0 * d0 + d1 * d1) + (d2 * d2 + d3 * d3);
    }
    if (tid == 0) submark(P, st, 0);
    const float2 mq = block_welford(C, m, M2, cols >> 7);   // one block reduction (R10)
    const float mu = mq.x, var = mq.y / (float)cols;
    const float rs = rsqrtf(var + st.eps);
    if (tid == 0) submark(P, st, 1);
    if (mine) {
      const float4 o = make_float4((v.x - mu) * rs * g.x + be.x, (v.y - mu) * rs * g.y + be.y,
                                   (v.z - mu) * rs * g.z + be.z, (v.w - mu) * rs * g.w + be.w);
      if (st.r_out_f) reinterpret_cast<float4*>(st.r_out_f + (int64_t)r * cols)[tid] = o;
      if (st.r_out_b)
        reinterpret_cast<uint2*>(st.r_out_b + (int64_t)r * cols)[tid] = make_uint2(pack_bf16(o.x, o.y), pack_bf16(o.z, o.w));
    }
    csync();   // C->red is reused by the next row of this CTA
  }
}

// ------------------------------------------------------------------ the persistent kernel
__global__ void __launch_bounds__(BERT_THREADS, 1) bert_kernel(const __grid_constant__ BertParams P) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  Ctrl* C = reinterpret_cast<Ctrl*>(smem);
  BStage* sbuf = reinterpret_cast<BStage*>(smem + 1024);   // two staged descriptors
  char* wring = smem + B_CTRL_BYTES;
  char* areg = wring + BW_SLOTS * BW_SLOT_BYTES;
  const int tid = threadIdx.x, warp = tid >> 5;
  if (tid == 0) {
    C->cur_stage = -1;
    for (int i = 0; i < BW_SLOTS; ++i) {
      ptx::mbar_init(&C->wfull[i], 1);
      ptx::mbar_init(&C->wempty[i], 1);
    }
    for (int i = 0; i < BA_SLOTS; ++i) {
      ptx::mbar_init(&C->afull[i], 1);
      ptx::mbar_init(&C->aempty[i], 1);
    }
    ptx::mbar_init(&C->accb, 1);
    ptx::mbar_init(&C->recvb, 1);
    ptx::mbar_init(&C->attb, 1);
    ptx::mbar_init(&C->qkvb, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 0) ptx::tmem_alloc(&C->tmem_base, 256);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  // the CTA pair (cluster) exchanges partial tiles through each other's shared memory: both CTAs
  // must have started and initialised their mbarriers before either sends (cluster barrier)
  if (P.pairs) {
    asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
    asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
  }

  if (warp == 8) {
    const int lane = tid & 31;
    if (lane == 0) weight_producer(P, C, wring);   // ---- weight producer
    if (lane == 1 && blockIdx.x == 0) ptx::prefetch_l2(P.stages, (uint32_t)(P.nstages * sizeof(BStage)));   // stage table
    return;
  }
  // ---- stage executor (warps 0-7).  Stage descriptors are double-buffered in smem: stage s+1's is
  // fetched while stage s runs, so it is never on the critical path behind a grid barrier.
  MmaState ms{0u, 0u, 0u, 0u, 0u, 0u, 0u};
  if (tid < (int)(sizeof(BStage) / 16))
    reinterpret_cast<int4*>(sbuf + (P.s_begin & 1))[tid] = __ldg(reinterpret_cast<const int4*>(P.stages + P.s_begin) + tid);
  csync();
  // Barrier participation: only the CTAs with work in stage s arrive at barrier s (its target is
  // st.workers), and a CTA waits for barrier s-1 only before a stage it works in.  Ordering stays
  // transitive because every stage has at least one worker, and each worker waited for the
  // previous barrier before its own arrival.
  int prev_workers = 0;
  // [s_begin, s_end) is the whole stage list except in the stage-isolation tests (debug)
  for (int s = P.s_begin; s < P.s_end; ++s) {
    const BStage& st = sbuf[s & 1];
    const bool work = has_work(P, st);
    if (work && s > P.s_begin) {
      if (st.fwait) flag_wait(P, st, st.kind == BS_ATTN ? (int)blockIdx.x % st.heads : (int)blockIdx.x % st.nsplit);
      else grid_wait(P, s - 1, prev_workers, st.kind != BS_ROW);
    }
    prev_workers = st.workers;
    // stage s+1's descriptor is copied by warp 7 (an epilogue-only warp in GEMM stages): thread 0 issues
    // the stage's first TMA / MMA and must not stall on this L2 load
    constexpr int kDescWarp = 7 * 32, kDescVecs = (int)(sizeof(BStage) / 16);
    if (s + 1 < P.s_end && tid >= kDescWarp && tid < kDescWarp + kDescVecs)
      reinterpret_cast<int4*>(sbuf + ((s + 1) & 1))[tid - kDescWarp] =
          __ldg(reinterpret_cast<const int4*>(P.stages + s + 1) + (tid - kDescWarp));
    if (tid == 0) {
      mark(P, s);
      C->cur_stage = s;
    }
    if (work) {
      if (!((P.dbg_skip >> st.kind) & 1)) {
        switch (st.kind) {
          case BS_GEMM: run_gemm(P, st, C, wring, areg, ms); break;
          case BS_ATTN: run_attn(P, st, C, wring, areg, ms); break;
          default:
            if (st.row_mode == 0) refresh_consts(P);
            run_row(P, st, C);
            break;
        }
      } else if ((st.kind == BS_GEMM || st.kind == BS_ATTN) && tid == 0) {
        // keep the weight ring in step with the producer: consume (and release) this task's groups
        const int nk = min(st.kchunks, st.K / 64 - (blockIdx.x % st.nsplit) * st.kchunks);
        const int gsz = wgroup(st.nt);
        for (int c0 = 0; c0 < nk; c0 += gsz, ++ms.wit) {
          const uint32_t slot = ms.wit % BW_SLOTS;
          ptx::mbar_wait(&C->wfull[slot], (ms.wit / BW_SLOTS) & 1);
          ptx::mbar_arrive(&C->wempty[slot]);
        }
      }
      if (tid == 0) submark(P, st, 6);
      if (st.arrive) grid_arrive(P, s, st.kind == BS_ROW || (st.kind == BS_GEMM && st.epi != EP_PARTIAL));
      if (tid == 0) submark(P, st, 7);
    }
    csync();   // descriptor s+1 visible; everyone is done with descriptor s
  }
  // ---- exit: the last CTA resets the barrier counters for the next launch
  csync();
  if (tid == 0) {
    __threadfence();
    const unsigned old = atomicAdd(&P.ctrl[P.nstages], 1u);
    if (old == gridDim.x - 1) {
      __threadfence();
      for (int k = 0; k <= P.nstages; ++k) P.ctrl[k] = 0u;
      for (int k = 0; k < P.nflags; ++k) P.ctrl[P.nstages + 1 + 32 * k] = 0u;
    }
  }
  if (P.prof && blockIdx.x == 0 && tid == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    P.prof[P.nstages + 1] = t;
  }
  ptx::tc_fence_before();
  csync();
  if (warp == 0) ptx::tmem_dealloc(C->tmem_base, 256);
}

}  // namespace bert

cudaError_t bert_launch(const BertParams& prm, int grid, bool pairs, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(bert::bert_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, B_SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(BERT_THREADS);
  cfg.dynamicSmemBytes = B_SMEM;
  cfg.stream = s;
  // Without clusters the launch is cooperative (the runtime checks co-residency).  With CTA pairs it
  // is a plain cluster launch whose co-residency bert_max_clusters() checked at plan time (a
  // cooperative cluster launch is refused under the profiler)
  cudaLaunchAttribute at[1];
  if (pairs) {
    at[0].id = cudaLaunchAttributeClusterDimension;   // CTA pairs (cluster-pair split-K stages)
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
  } else {
    at[0].id = cudaLaunchAttributeCooperative;
    at[0].val.cooperative = 1;
  }
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, bert::bert_kernel, prm);
}

// how many CTA-pair clusters of the BERT kernel can be resident at once (all must be: spin barriers)
cudaError_t bert_max_clusters(int grid, int* clusters) {
  cudaError_t e = cudaFuncSetAttribute(bert::bert_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, B_SMEM);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(bert::bert_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 0);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(BERT_THREADS);
  cfg.dynamicSmemBytes = B_SMEM;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 2;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaOccupancyMaxActiveClusters(clusters, bert::bert_kernel, &cfg);
}

cudaError_t bert_max_active(int* blocks) {
  cudaError_t e = cudaFuncSetAttribute(bert::bert_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, B_SMEM);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, bert::bert_kernel, BERT_THREADS, B_SMEM);
}

}  // namespace souffle
