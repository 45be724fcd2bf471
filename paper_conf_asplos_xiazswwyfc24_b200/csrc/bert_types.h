// Plain-data structures shared by the host planner (csrc/host/bert.cpp) and the specialised
// BERT-encoder subprogram kernel (csrc/kernels/bert.cu).
//
// When the partitioned TE program is a stack of BERT encoder layers (Table 2,
// 49 TEs per layer), the whole program is one subprogram (§5.4) and is run
// by one persistent cooperative kernel whose stages are the fused patterns of §6:
//   GEMM  horizontal / plain tcgen05 GEMM (§6.1).  Epilogues (vertical transformation §6.2):
//           EP_QKV     + bias, bf16, the reshape/permute index map folded into the store
//                      (Q, K head-major [2*heads][S][d]; V transposed [heads][d][S])
//           EP_GELU    + bias, erf-GELU, bf16 [S][N]
//           EP_PARTIAL split-K partial, fp32 [split][S][N] plain stores (summed by the consumer)
//   ATTN  per head: QK^T -> scale -> max-subtracted softmax -> PV, S and O in TMEM (Fig. 1(c))
//   ROW   per token row: sum of split-K partials + bias + residual + LayerNorm ((mean, M2) merged
//         pairwise from exactly centred per-thread values, so a constant row gives beta), fp32 and bf16
//         outputs (the two-phase reduction of P:L527-536).  Stage 0 (row_mode 0) converts the fp32
//         input to bf16 and, on all CTAs, refreshes the packed constant vectors from the bound
//         pointers.
// Weights never depend on activations, so a producer warp streams every GEMM stage's weight tiles
// through a shared-memory ring ahead of the grid barriers (§6.5 "cross-stage prefetch").
#pragma once
#include <stdint.h>

namespace souffle {

enum BStageKind : int32_t { BS_GEMM = 0, BS_ATTN = 1, BS_ROW = 2 };
enum BEpilogue : int32_t { EP_PARTIAL = 0, EP_QKV = 1, EP_GELU = 2 };

enum {
  BERT_THREADS = 288,          // 8 compute warps + 1 weight-producer warp
  BERT_COMPUTE = 256,
  BW_SLOTS = 5,                // weight ring: 5 x 16 KB; a slot holds 16 KB / (n_tile * 128 B) K-chunks
  BW_SLOT_BYTES = 16384,
  BA_SLOTS = 7,                // A operand ring: 7 x (128 rows x 64 K bf16) >= the 6 K chunks a
                               // cluster-pair task streams; also the attention operands and staging
  BA_SLOT_BYTES = 16384,
  B_CTRL_BYTES = 2048,         // control block + two staged stage descriptors
  B_AREGION = BA_SLOTS * BA_SLOT_BYTES,   // also holds the attention operands Q, K, V^T, P (80 KB)
  B_RECV_BYTES = 16384,        // cluster-pair split-K: the partner's fp32 half tile (128 x <= 32 cols)
  B_SMEM = B_CTRL_BYTES + BW_SLOTS * BW_SLOT_BYTES + B_AREGION + B_RECV_BYTES + 1024   // + alignment slack
};

struct alignas(16) BStage {
  int32_t kind, ntasks, layer, idx;   // idx: position in the stage list
  // ---- GEMM: task = tile * nsplit + split; each split covers kchunks chunks of 64 along K
  int32_t nt, tiles_n, nsplit, kchunks;
  int32_t K, N, wmap0, wrows;   // W tensor maps wmap0.. (an N tile never straddles two maps)
  int32_t amap, epi, heads, workers;   // workers: CTAs with work in this stage (barrier arrivals)
  const float* bias;            // EP_QKV / EP_GELU: fp32 [N]
  float* part;                  // EP_PARTIAL: fp32 [nsplit][S][N]
  uint16_t* out_b;              // EP_GELU: bf16 [S][N];  EP_QKV: Q,K [2*heads][S][64]
  uint16_t* out_vt;             // EP_QKV: V^T [heads][64][S]
  // ---- ATTN: TMA maps of Q/K ([2*heads][S][64]) and V^T ([heads][64][S])
  int32_t qkmap, vtmap, d, H;
  uint16_t* ctx;                // bf16 [S][H], head h at columns h*64 ..
  float scale, eps;
  // ---- point-to-point dependencies (instead of a grid barrier; §6.4 only needs a global sync for
  // one-relies-on-many edges).  A consumer stage with fwait waits until flag fin[idx] reaches fneed
  // (idx = head for ATTN, K split for a GEMM); a producer stage with fout adds 1 to
  // fout[(n0 % fmod) / fdiv] after its epilogue.  Flags are 128 B apart.  arrive: the next stage
  // waits on this stage's grid barrier.
  int32_t fwait, fneed, fdiv, fmod;
  unsigned int* fin;
  unsigned int* fout;
  // ---- ROW: mode 0 convert (out_b = bf16(in)); mode 1 LayerNorm(sum_s part[s] + bias + res)
  int32_t row_mode, cols, r_nsplit, arrive;
  int32_t cpair, pad0, pad1, pad2;   // GEMM nsplit == 2 over a CTA pair (cluster): partial sums
                                     // exchanged through distributed shared memory (DSMEM)
  const float* r_in;            // mode 0: fp32 [S][cols]; mode 1: partials [r_nsplit][S][cols]
  const float* r_bias;
  const float* r_res;
  const float* r_gamma;
  const float* r_beta;
  float* r_out_f;
  uint16_t* r_out_b;
};

// one constant vector (bias / gamma / beta) refreshed from its bound pointer into the packed
// workspace copy by stage 0 of every launch (so an in-place update of a bound parameter is seen)
struct alignas(16) BCopy {
  const float* src;
  float* dst;
  int32_t n, first;             // first: flat index of element 0 in the concatenation of all vectors
};

struct BertParams {
  const BStage* stages;
  const void* tmaps;            // CUtensorMap[] (128 B each)
  unsigned int* ctrl;           // [0, nstages): per-barrier arrival counters; [nstages]: exit counter;
                                // [nstages + 1 + 32 k]: point-to-point flag k (nflags of them)
  unsigned long long* prof;     // optional per-stage %globaltimer marks, null if off
  int32_t nstages, S;
  int32_t dbg_skip;             // debug: bit k set -> stages of kind k do no work (barriers only)
  int32_t nflags;
  const BCopy* copies;          // constant vectors refreshed in stage 0 (all CTAs take part)
  int32_t ncopies, copy_total;  // entries, total floats
  int32_t s_begin, s_end;       // stages executed: [0, nstages) except in stage-isolation tests
  int32_t pairs;                // launched as CTA-pair clusters (cluster-pair split-K stages)
};

}  // namespace souffle
