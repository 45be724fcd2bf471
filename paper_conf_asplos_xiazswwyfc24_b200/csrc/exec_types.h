// Plain-data structures shared by the host lowering (csrc/host/lower.cpp) and the sm_100a
// executor (csrc/kernels/exec.cu).  A lowered subprogram is a list of Stages executed by ONE
// persistent cooperative kernel, with a grid barrier before every stage that depends on an
// earlier one (§6.4: "inserts global sync primitives between TEs with
// one-relies-on-many dependency"; Fig. 2).
#pragma once
#include <stdint.h>

namespace souffle {

enum StageKind : int32_t {
  ST_EW = 0,        // vertically fused one-relies-on-one chain over a 2-D domain (§6.2)
  ST_REDUCE = 1,    // one reduction TE with fused producer (pre) and consumer (post) chains
  ST_GEMM_SIMT = 2, // fp32 / small / batched matmuls (horizontal members), fused epilogue
  ST_GEMM_TC = 3,   // bf16 tcgen05 GEMM, TMA-fed, split-K with last-arriver epilogue
  ST_ATTN = 4       // QK^T -> scale -> softmax -> PV pattern, tcgen05 (fused reductions, §2.3)
};

// Instruction set of the fused-chain interpreter.  Registers are vectors of W columns.
enum OpCode : int16_t {
  OP_LOAD = 0,   // R[a] = load(addr)
  OP_ACC = 1,    // R[a] = accumulator (GEMM / reduction result)
  OP_UN = 2,     // R[a] = fn(R[a])
  OP_BIN = 3,    // R[a] = fn(R[a], R[b])
  OP_BINL = 4,   // R[a] = fn(R[a], load(addr)), b != 0: fn(load(addr), R[a])
  OP_SCAL = 5,   // R[a] = fn(R[a], imm)
  OP_STORE = 6,  // store R[a] -> addr (dtype of addr)
  OP_MOV = 7,    // R[a] = R[b]
  OP_RED = 8,    // red[b] += sum_cols(R[a]) * imm ; flushed to addr(row, 0) with atomics (§6.3)
  OP_BINR = 9    // R[a] = fn(R[b], R[a])   (operands evaluated in Sethi-Ullman order)
};

enum Fn : int16_t {
  FN_ADD = 0, FN_SUB = 1, FN_MUL = 2, FN_DIV = 3, FN_MAX = 4,
  FN_EXP = 5, FN_TANH = 6, FN_SIGMOID = 7, FN_RELU = 8, FN_GELU = 9, FN_RSQRT = 10, FN_NEG = 11,
  FN_ADDS = 12, FN_MULS = 13
};

enum { NREG = 4, CHUNK = 8, MAX_RED = 4, MAX_BUFS = 480, EXEC_THREADS = 256, EXEC_SMEM = 136 * 1024 };

// Software-managed shared-memory tensor cache (§6.5, "tensor reuse
// optimization"): fp32 words above the EXEC_SMEM working area, so GEMM / attention stages between a
// tensor's producer and its consumers leave it intact.  At most EXEC_CACHE_FLOATS (88 KB: a CTA stays
// within the 227 KB opt-in limit); by default EXEC_CACHE_DEFAULT_FLOATS (24 KB), which still fits the
// 164 KB shared-memory carveout the working area needs -- a larger cache shrinks L1, which the
// interpreter's index-table and weight loads use (measured on Swin-B / BERT V3).
enum { EXEC_CACHE_FLOATS = 22528, EXEC_CACHE_DEFAULT_FLOATS = 6144 };
enum CacheMode : int16_t { CM_FILL = 1, CM_NOSTORE = 2 };

// Address of a tensor element at domain point (r, c):
//   element offset = base + row(r) + col(c)
//   mode 0 affine:    row(r) = r*rs,            col(c) = c*cs
//   mode 1 separable: row(r) = tab[rtab + r],   col(c) = tab[ctab + c]
//   mode 2 full:      row(r) + col(c) = tab[ftab + r*ncols + c]
struct Addr {
  uint64_t ptr;   // resolved at souffle_workspace_init: address of element `base` (device uses ptr +
                  // element offset of row(r) + col(c); `buf`/`base` are the host-side description)
  int64_t base;
  int64_t rs, cs;
  int32_t buf;    // >= 0: bound pointer table index; -1: workspace (base counted from ws_data)
  int32_t dtype;  // 0 f32, 1 bf16
  int32_t mode;
  int32_t rtab, ctab, ftab, ncols;
  int16_t cg;     // 1: tensor is written inside the run -> coherent (L2) loads
  int16_t cvec;   // mode 1: col(c0 + j) == col(c0) + j within every aligned chunk of CHUNK columns
  // tensor cache (row-block stages, mode 0 only): cache = float offset of the tensor's slot in the
  // cache region + 1 (0: not cached).  Domain row r belongs to row block r / crb, which CTA
  // (r / crb) % gridDim.x owns in every row-block stage of the launch; element (r, c) lives at
  // slot + ((r / crb) / gridDim.x) * crb * rs + (r % crb) * rs + c * cs.  A load reads the slot
  // (cmode & CM_FILL: reads global memory and deposits the chunk); a store writes the slot, rounded
  // to dtype, and global memory unless cmode & CM_NOSTORE (every consumer hits).
  int32_t cache;
  int16_t crb, cmode;
};

struct Ins {
  int16_t op, a, b, fn;
  int32_t addr;
  float imm;
};

// A fused-chain program: Ins[ins0 .. ins0+len) whose Ins.addr index a program-local Addr table
// addrs[addr0 .. addr0+naddr).  Programs and their tables are small enough to be staged in
// shared memory once per stage / task, so the interpreter never chases global pointers.
// Compiled fast paths the host recognises in a program (all fields are instruction indices whose
// `addr` is used, or -1).  kind 1 "linear epilogue": v = act(acc + side0 + side1); store v to st0 /
// st1; row sums of v and v*v into red_sum / red_sq.  kind 2 "LayerNorm apply" (EW domain):
// v = (x - mu) * rsqrt(msq - mu*mu + eps) * g + b; store to st0 / st1.  kind 0: interpret.
struct FastPath {
  int32_t kind;
  int32_t side0, side1, act;
  int32_t st0, st1, red_sum, red_sq;
  int32_t ln_x, ln_mu, ln_msq, ln_g, ln_b;
  float eps;
  float red_scale_sum, red_scale_sq;
};

struct ProgRef {
  int32_t ins0, len, addr0, naddr;
  FastPath fast;
};

struct GemmMember {
  int32_t M, N, K, batch;   // domain rows = batch*M (b-major), cols = N
  int32_t prec;             // SIMT: 1 -> round operands to bf16
  int32_t a_addr, b_addr;   // SIMT: A at (r = b*M+m, c = k), B at (r = b*N+n, c = k)
  ProgRef prog;             // epilogue program at (r, c)
  int32_t tiles_m, tiles_n, splits, task0;  // tasks = tiles_m*tiles_n*splits, starting at task0
  int32_t n_tile, k_split;  // TC: N tile, K per split (multiple of 64)
  int32_t a_tmap, b_tmap;   // TC: TMA descriptor indices (a_tmap < 0 -> manual fp32 A path)
  int32_t a_f32;            // TC manual path: Addr of fp32 A, rows contiguous with stride K
  int32_t acc_off;          // TC split-K: workspace float offset of the fp32 accumulator
  int32_t cnt_off;          // TC split-K: workspace u32 offset of per-tile arrival counters
  int32_t gemv;             // SIMT: 1 -> skinny GEMM (few rows): a warp per output element,
                            // lanes split K; task = 8 consecutive (row, col) outputs
};

struct Stage {
  int32_t kind, barrier_before, ntasks, sp;
  int32_t rows, cols;               // EW / REDUCE domain
  ProgRef prog;                     // EW program; REDUCE pre-program at (o, e); ATTN epilogue
  ProgRef post;                     // REDUCE post-program at (o, 0)
  int32_t red_fn;                   // REDUCE: 0 sum, 1 max
  float red_scale;                  // REDUCE: 1/E for mean
  int32_t mem0, nmem;               // GEMM members
  // ATTN: q/k/v are bf16 [B, S, d] contiguous workspace tensors
  int32_t at_B, at_S, at_d, at_q, at_k, at_v;  // q/k/v: Addr index (base, buf used)
  float at_scale;
  int32_t barrier_after;            // the next stage of the same launch starts with a grid barrier
  int32_t at_add[2];                // ATTN: Addr of additive score terms at (b*S + i, j), -1 if none
  // REDUCE / EW: rows per row block.  CTA b owns row blocks b, b + grid, ... (REDUCE: always, a warp
  // per 32/G rows; EW: when rblk > 0, else chunk t goes to thread t mod (grid * threads)).  Stages
  // of one launch with equal rows and rblk hand rows to the same CTA: a dependency between them is
  // CTA-local (no grid barrier, tensor cache hits).
  int32_t rblk;
  int32_t pad_rb[3];
};

struct Launch {
  int32_t first, count;   // stage range
  int32_t grid, cooperative, uses_tc, is_last;
  int32_t smem;
  int32_t nbarriers;
};

// kernel parameter block (passed by value; <= 32 KB param limit on sm_70+ / CUDA 12.1+)
struct Params {
  const Stage* stages;
  const GemmMember* members;
  const Ins* ins;
  const Addr* addrs;
  const int32_t* tabs;
  const void* tmaps;          // CUtensorMap[] (64 B aligned, global memory)
  char* ws_data;              // intermediates / accumulators
  unsigned int* ctrl;         // [0] barrier counter, [1] exit counter
  const int64_t* zero_list;   // (byte offset, bytes) pairs in ws_data, zeroed by the last CTA
  unsigned long long* prof;   // optional: %globaltimer at every stage start (CTA 0), null if off;
                              // followed by 8 sub-stage marks per stage (prof[nst + 1 + 8*s + k])
  int32_t n_stages_total;
  int32_t n_zero;
  int32_t first, count, cooperative, uses_tc, is_last;
  unsigned int* progress;     // per-CTA (stage << 8 | point) of thread 0, read by the watchdog
  void* bufs[MAX_BUFS];
};

}  // namespace souffle
