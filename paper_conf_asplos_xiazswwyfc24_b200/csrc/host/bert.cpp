// BERT encoder-stack pattern: strict TE-pattern match, tile policy, workspace layout, stage table
// and launch of the specialised persistent kernel (kernels/bert.cu).
//
// Pattern (SURVEY.md Appendix A, 49 TEs per layer; Table 2, Fig. 1):
//   Q/K/V = X Wᵀ + b (three matmuls sharing X: one horizontal group, §6.1)
//   reshape [S,nh,d] + permute (1,0,2)      (OR index maps, folded into the attention loads, §6.2)
//   softmax(Q Kᵀ · 1/√d) V                  (max-subtracted; reductions fused, §2.3)
//   permute + reshape back, Wo, +bo, +X     (residual)
//   LayerNorm (mean, sub, square, mean, +eps, rsqrt, mul, ×γ, +β)
//   W1, +c1, GELU(erf), W2, +c2, +L1, LayerNorm
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <sstream>
#include <string>

#include <cuda.h>
#include <cuda_runtime.h>

#include "../bert_types.h"
#include "plan.h"

namespace souffle {

extern thread_local std::string g_err;
souffle_status fail(souffle_status c, const std::string& m);
cudaError_t bert_launch(const BertParams& prm, int grid, bool pairs, cudaStream_t s);
cudaError_t bert_max_active(int* blocks);
cudaError_t bert_max_clusters(int grid, int* clusters);

namespace {

struct Cursor {
  const Graph& g;
  size_t i = 0;
  bool ok = true;
  explicit Cursor(const Graph& gr) : g(gr) {}
  const Node* next(int op) {
    if (!ok || i >= g.nodes.size() || g.nodes[i].op != op) { ok = false; return nullptr; }
    return &g.nodes[i++];
  }
  int id() const { return (int)i - 1; }
  int ph(std::vector<int64_t> shape, int dtype) {
    const Node* n = next(SOUFFLE_OP_PLACEHOLDER);
    if (!n || !n->is_const || n->shape != shape || n->dtype != dtype) { ok = false; return -1; }
    return id();
  }
  int mm(int a, int b, int trans) {
    const Node* n = next(SOUFFLE_OP_MATMUL);
    if (!n || n->a != a || n->b != b || n->trans_b != trans || n->prec != SOUFFLE_BF16) { ok = false; return -1; }
    return id();
  }
  int ew(int fn, std::vector<int> in) {
    const Node* n = next(SOUFFLE_OP_ELEMENTWISE);
    if (!n || n->fn != fn || n->in != in) { ok = false; return -1; }
    return id();
  }
  int ews(int fn, int in, double* scalar) {
    const Node* n = next(SOUFFLE_OP_ELEMENTWISE);
    if (!n || n->fn != fn || n->in.size() != 1 || n->in[0] != in) { ok = false; return -1; }
    *scalar = n->scalar;
    return id();
  }
  int red(int fn, int in, int axis) {
    const Node* n = next(SOUFFLE_OP_REDUCE);
    if (!n || n->fn != fn || n->in[0] != in || n->axis != axis || !n->keepdim) { ok = false; return -1; }
    return id();
  }
  int reshape(int in, std::vector<int64_t> shape) {
    const Node* n = next(SOUFFLE_OP_RESHAPE);
    if (!n || n->in[0] != in || n->shape != shape) { ok = false; return -1; }
    return id();
  }
  int permute(int in, std::vector<int> perm) {
    const Node* n = next(SOUFFLE_OP_PERMUTE);
    if (!n || n->in[0] != in || n->perm != perm) { ok = false; return -1; }
    return id();
  }
};

// LayerNorm chain of SURVEY Appendix A ids 25-33 / 40-48; returns the output id
int match_ln(Cursor& c, int x, int64_t H, int* gamma, int* beta, double* eps) {
  int mu = c.red(SOUFFLE_RED_MEAN, x, 1);
  int d = c.ew(SOUFFLE_EW_SUB, {x, mu});
  int q = c.ew(SOUFFLE_EW_MUL, {d, d});
  int v = c.red(SOUFFLE_RED_MEAN, q, 1);
  int ve = c.ews(SOUFFLE_EW_ADD_SCALAR, v, eps);
  int rs = c.ew(SOUFFLE_EW_RSQRT, {ve});
  int n = c.ew(SOUFFLE_EW_MUL, {d, rs});
  *gamma = c.ph({H}, SOUFFLE_F32);
  int a = c.ew(SOUFFLE_EW_MUL, {n, *gamma});
  *beta = c.ph({H}, SOUFFLE_F32);
  return c.ew(SOUFFLE_EW_ADD, {a, *beta});
}

bool match_layer(Cursor& c, int X, BertPlan& bp, BertLayerIds& L, double* eps1, double* eps2) {
  const int64_t S = bp.S, H = bp.H, nh = bp.heads, d = bp.d;
  int qkv[3], W[3], b[3];
  for (int k = 0; k < 3; ++k) {
    W[k] = c.ph({H, H}, SOUFFLE_BF16);
    int m = c.mm(X, W[k], 1);
    b[k] = c.ph({H}, SOUFFLE_F32);
    qkv[k] = c.ew(SOUFFLE_EW_ADD, {m, b[k]});
  }
  int p[3];
  for (int k = 0; k < 3; ++k) p[k] = c.permute(c.reshape(qkv[k], {S, nh, d}), {1, 0, 2});
  int Sc = c.mm(p[0], p[1], 1);
  double sc = 0;
  int Ss = c.ews(SOUFFLE_EW_MUL_SCALAR, Sc, &sc);
  if (c.ok && std::fabs(sc - 1.0 / std::sqrt((double)d)) > 1e-12) c.ok = false;
  int Mx = c.red(SOUFFLE_RED_MAX, Ss, 2);
  int Sd = c.ew(SOUFFLE_EW_SUB, {Ss, Mx});
  int E = c.ew(SOUFFLE_EW_EXP, {Sd});
  int Z = c.red(SOUFFLE_RED_SUM, E, 2);
  int P = c.ew(SOUFFLE_EW_DIV, {E, Z});
  int Cx = c.mm(P, p[2], 0);
  int Cr = c.reshape(c.permute(Cx, {1, 0, 2}), {S, H});
  L.Wo = c.ph({H, H}, SOUFFLE_BF16);
  int A0 = c.mm(Cr, L.Wo, 1);
  L.bo = c.ph({H}, SOUFFLE_F32);
  int R1 = c.ew(SOUFFLE_EW_ADD, {c.ew(SOUFFLE_EW_ADD, {A0, L.bo}), X});
  int L1 = match_ln(c, R1, H, &L.g1, &L.be1, eps1);
  L.W1 = c.ph({bp.F, H}, SOUFFLE_BF16);
  int F0 = c.mm(L1, L.W1, 1);
  L.c1 = c.ph({bp.F}, SOUFFLE_F32);
  int F2 = c.ew(SOUFFLE_EW_GELU_ERF, {c.ew(SOUFFLE_EW_ADD, {F0, L.c1})});
  L.W2 = c.ph({H, bp.F}, SOUFFLE_BF16);
  int O0 = c.mm(F2, L.W2, 1);
  L.c2 = c.ph({H}, SOUFFLE_F32);
  int R2 = c.ew(SOUFFLE_EW_ADD, {c.ew(SOUFFLE_EW_ADD, {O0, L.c2}), L1});
  L.out = match_ln(c, R2, H, &L.g2, &L.be2, eps2);
  L.Wq = W[0]; L.Wk = W[1]; L.Wv = W[2];
  L.bq = b[0]; L.bk = b[1]; L.bv = b[2];
  return c.ok;
}

// Tile policies (performance policies, not semantics).
// Full-K GEMM (fused bias / GELU / QKV-scatter epilogue): the smallest N tile (more CTAs streaming
// weights, less weight per CTA) whose tiles fit one wave; every task reads the whole A operand
// through the 5-slot TMA ring.
BertGemmCfg full_cfg(int64_t N, int64_t K, int sms, int max_nt, const char* env) {
  BertGemmCfg c;
  for (int nt : {16, 32, 64, 128}) {
    if (nt > max_nt || N % nt) continue;
    if (c.nt == 0 || N / nt <= sms) c = BertGemmCfg{nt, 1, (int)(K / 64), (int)(N / nt)};
    if (N / nt <= sms) break;
  }
  if (const char* e = std::getenv(env)) {
    int nt = 0;
    // the kernel's epilogues exist for n tiles of 16, 32, 64 and 128 only (max_nt: QKV tiles must not
    // straddle a 64-wide head)
    if (std::sscanf(e, "%d", &nt) == 1 && (nt == 16 || nt == 32 || nt == 64 || nt == 128) && nt <= max_nt &&
        N % nt == 0 && N / nt <= sms)
      c = BertGemmCfg{nt, 1, (int)(K / 64), (int)(N / nt)};
  }
  return c;
}
// Split-K GEMM whose fp32 partials are summed by the LayerNorm row stage: minimise the bytes on the
// critical path of one task (A chunks + partial tile) plus what each LayerNorm row reads back
// (nsplit partial rows), within one wave of CTAs.
BertGemmCfg split_cfg(int64_t N, int64_t K, int sms, const char* env) {
  BertGemmCfg best;
  const int kc = (int)(K / 64);
  double best_cost = 1e30;
  for (int nt : {16, 32, 64, 128}) {
    if (N % nt) continue;
    const int tiles = (int)(N / nt);
    for (int kch = 1; kch <= kc; ++kch) {
      const int nsplit = (kc + kch - 1) / kch;
      if ((int64_t)tiles * nsplit > sms || nsplit > 12) continue;   // kMaxSplit in kernels/bert.cu
      const double cost = kch * 16384.0 + 128.0 * nt * 4 + nsplit * N * 4.0;
      if (cost < best_cost - 1) {
        best_cost = cost;
        best = BertGemmCfg{nt, nsplit, kch, tiles};
      }
    }
  }
  if (const char* e = std::getenv(env)) {   // SOUFFLE_BERT_<STAGE>=nt,kchunks
    int nt = 0, kch = 0;
    if (std::sscanf(e, "%d,%d", &nt, &kch) == 2 && (nt == 16 || nt == 32 || nt == 64 || nt == 128) && N % nt == 0 &&
        kch >= 1) {
      const int nsplit = (kc + kch - 1) / kch;
      if ((int64_t)(N / nt) * nsplit <= sms && nsplit <= 12) best = BertGemmCfg{nt, nsplit, kch, (int)(N / nt)};
    }
  }
  return best;
}

int64_t al(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

// activation tensor maps: xb, ctx, l1b, h (A operands), Q/K (3-D), V^T (3-D); then 6 W maps per layer
enum { MAP_XB = 0, MAP_CTX = 1, MAP_L1B = 2, MAP_H = 3, MAP_QK = 4, MAP_VT = 5, kActMaps = 6 };

}  // namespace

void bert_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, BertPlan& bp) {
  bp = BertPlan();
  auto no = [&](const char* why) { bp.on = false; bp.why_not = why; };
  if (flags != 0) return no("ablation flags select the generic executor");
  const auto& N = g.nodes;
  if (N.empty() || N[0].op != SOUFFLE_OP_PLACEHOLDER || N[0].is_const || N[0].dtype != SOUFFLE_F32 ||
      N[0].shape.size() != 2)
    return no("first node is not an fp32 [S, H] input");
  bp.X = 0;
  bp.S = (int)N[0].shape[0];
  bp.H = (int)N[0].shape[1];
  // heads / FFN width from the first layer's reshape and W1 (probe, then strict match)
  if (N.size() < 20) return no("too small");
  int nh = 0;
  for (const Node& n : N)
    if (n.op == SOUFFLE_OP_RESHAPE && n.shape.size() == 3) { nh = (int)n.shape[1]; break; }
  if (nh <= 0) return no("no head reshape");
  bp.heads = nh;
  bp.d = bp.H / nh;
  for (const Node& n : N)
    if (n.op == SOUFFLE_OP_PLACEHOLDER && n.is_const && n.shape.size() == 2 && n.shape[1] == bp.H && n.shape[0] != bp.H) {
      bp.F = (int)n.shape[0];
      break;
    }
  if (bp.S < 1 || bp.S > 128) return no("S must be in [1, 128] (one M=128 tcgen05 tile)");
  if (bp.d != 64 || bp.H % 128 || bp.H > 768) return no("needs head dim 64 and H a multiple of 128 (<= 768)");
  if (bp.F <= 0 || bp.F % 128 || bp.F > 8192) return no("FFN width must be a multiple of 128");
  if (nh * 64 != bp.H) return no("H != heads * 64");
  Cursor c(g);
  c.i = 1;
  int x = 0;
  double eps = -1;
  while (c.ok && c.i < N.size()) {
    BertLayerIds L;
    double e1 = 0, e2 = 0;
    if (!match_layer(c, x, bp, L, &e1, &e2)) break;
    if (eps < 0) eps = e1;
    if (e1 != eps || e2 != eps) { c.ok = false; break; }
    bp.layers.push_back(L);
    x = L.out;
  }
  if (!c.ok || bp.layers.empty()) return no("TE program is not a BERT encoder stack");
  if (g.outputs.size() != 1 || g.outputs[0] != x) return no("the only output must be the last layer's LayerNorm");
  // driven by the partition: one subprogram (one persistent launch), and per layer the QKV GEMM is the
  // analysis' N-concat horizontal group of the three matmuls that read the layer input
  if (an.num_sp != 1) return no("the partition has more than one subprogram");
  for (size_t i = 0; i < g.nodes.size(); ++i)
    if (g.nodes[i].op != SOUFFLE_OP_PLACEHOLDER && an.assign[i] != 0) return no("TE outside subprogram 0");
  for (const BertLayerIds& L : bp.layers) {
    int mm[3], k = 0;
    for (size_t i = 0; i < g.nodes.size() && k < 3; ++i)
      if (g.nodes[i].op == SOUFFLE_OP_MATMUL && (g.nodes[i].b == L.Wq || g.nodes[i].b == L.Wk || g.nodes[i].b == L.Wv))
        mm[k++] = (int)i;
    if (k != 3) return no("QKV matmuls");
    const int gid = an.hgid[mm[0]];
    if (gid < 0 || an.hgid[mm[1]] != gid || an.hgid[mm[2]] != gid || an.hkind[gid] != 0)
      return no("the analysis did not group Q, K, V into one N-concat horizontal GEMM (§6.1)");
  }
  bp.eps = eps;
  bp.Y = x;
  bp.num_sms = dev.num_sms > 0 ? dev.num_sms : 148;
  const int sms = bp.num_sms;
  if (bp.S % 8) return no("S must be a multiple of 8 (V^T rows are TMA-loaded)");
  if (bp.H > 768) return no("hidden size must be <= 768 (at most 12 heads of 64: split-K partials per LayerNorm row)");
  bp.qkv = full_cfg(3LL * bp.H, bp.H, sms, 64, "SOUFFLE_BERT_QKV");     // tiles never straddle a head
  // out-projection fused into attention: split-K over heads (K = 64 per head), N tiles of nt rows
  bp.out = BertGemmCfg{};
  for (int nt : {16, 32, 64, 128})
    if (bp.H % nt == 0 && (bp.H / nt) * bp.heads <= sms) { bp.out = BertGemmCfg{nt, bp.heads, 1, bp.H / nt}; break; }
  if (bp.heads > 12) return no("more than 12 heads (split-K partials summed per LayerNorm row)");
  bp.ffn1 = full_cfg(bp.F, bp.H, sms, 128, "SOUFFLE_BERT_FFN1");
  // cluster-pair split-K for the full-K GEMMs (QKV, FFN1): a CTA pair splits K in halves and sums
  // through DSMEM, halving the activation bytes every CTA streams (SOUFFLE_BERT_PAIRS=0 disables)
  {
    const char* e = std::getenv("SOUFFLE_BERT_PAIRS");
    const int kc = bp.H / 64;
    bp.pairs = (!e || std::atoi(e) != 0) && sms % 2 == 0 && kc % 2 == 0;
    if (bp.pairs) {
      int qn = 32, fn = 64;   // N tiles of the pair GEMMs (SOUFFLE_BERT_PAIR_NT=qkv,ffn1 for tile studies)
      if (const char* t = std::getenv("SOUFFLE_BERT_PAIR_NT")) {
        int a = 0, b = 0;
        if (std::sscanf(t, "%d,%d", &a, &b) == 2 && (a == 32 || a == 64) && (b == 32 || b == 64)) { qn = a; fn = b; }
      }
      const BertGemmCfg q{qn, 2, kc / 2, (int)(3 * bp.H / qn)}, f{fn, 2, kc / 2, (int)(bp.F / fn)};
      if (q.tiles_n * 2 <= sms && f.tiles_n * 2 <= sms) {
        bp.qkv = q;
        bp.ffn1 = f;
      } else {
        bp.pairs = false;
      }
    }
  }
  bp.ffn2 = split_cfg(bp.H, bp.F, sms, "SOUFFLE_BERT_FFN2");
  for (const BertGemmCfg* q : {&bp.qkv, &bp.out, &bp.ffn1, &bp.ffn2})
    if (q->nt == 0 || q->tiles_n * q->nsplit > sms) return no("no tile configuration fits one wave of CTAs");
  bp.nstages = 1 + 6 * (int)bp.layers.size();
  // ---- workspace layout
  int64_t o = 0;
  bp.nflags = (int)bp.layers.size() * (bp.heads + bp.ffn2.nsplit);
  bp.o_ctrl = o; o = al(o + 4 * (bp.nstages + 2 + 32 * (int64_t)bp.nflags), 256);
  bp.o_prof = o; o = al(o + 8 * (17 * bp.nstages + 2), 256);
  bp.o_stages = o; o = al(o + (int64_t)sizeof(BStage) * bp.nstages, 256);
  bp.o_tmaps = o; o = al(o + 128 * (kActMaps + 6 * (int64_t)bp.layers.size()), 256);
  const int64_t S = bp.S, H = bp.H, F = bp.F;
  auto take = [&](int64_t bytes) { int64_t r = o; o = al(o + bytes, 1024); return r; };
  bp.o_xb = take(S * H * 2);
  bp.o_ctx = take(S * H * 2);
  bp.o_l1b = take(S * H * 2);
  bp.o_l1f = take(S * H * 4);
  bp.o_xf = take(S * H * 4);
  bp.o_h = take(S * F * 2);
  bp.o_qk = take(2 * S * H * 2);
  bp.o_vt = take(S * H * 2);
  bp.o_part_o = take((int64_t)bp.out.nsplit * S * H * 4);
  bp.o_part_2 = take((int64_t)bp.ffn2.nsplit * S * H * 4);
  // all small per-layer vectors packed contiguously (a handful of 2 MB pages instead of ~200
  // scattered allocations: every TLB miss is a microsecond on the critical path)
  bp.o_consts = take((int64_t)bp.layers.size() * (9 * H + F) * 4);
  bp.o_copies = take((int64_t)bp.layers.size() * 10 * (int64_t)sizeof(BCopy));
  bp.total = al(o, 4096);
  bp.on = true;
}

std::string bert_describe(const BertPlan& bp) {
  std::ostringstream os;
  if (!bp.on) {
    os << "pattern bert: not used (" << bp.why_not << ")\n";
    return os.str();
  }
  auto g = [&](const char* nm, const BertGemmCfg& c) {
    const bool pair = bp.pairs && (&c == &bp.qkv || &c == &bp.ffn1);
    os << "    " << nm << ": n_tile " << c.nt << " x split-K " << c.nsplit << " (" << c.kchunks * 64
       << " K per task) = " << c.tiles_n * c.nsplit << " tasks" << (pair ? " (cluster pairs, DSMEM reduction)" : "")
       << "\n";
  };
  os << "pattern bert: " << bp.layers.size() << " encoder layer(s), S=" << bp.S << " H=" << bp.H << " heads="
     << bp.heads << " F=" << bp.F << " -> 1 persistent launch (kernels/bert.cu), " << bp.nstages << " stages, "
     << bp.nstages - 1 << " grid barriers\n";
  os << "  per layer: QKV-gemm(+bias, head-major Q/K, V^T) | attention+out-proj(" << bp.heads << " heads x "
     << bp.out.tiles_n << " N tiles, split-K partials) | LN1-row | FFN1-gemm(+bias, GELU) | FFN2-gemm(split-K "
        "partials) | LN2-row\n";
  g("qkv ", bp.qkv);
  g("attn-out", bp.out);
  g("ffn1", bp.ffn1);
  g("ffn2", bp.ffn2);
  return os.str();
}

// ------------------------------------------------------------------ runtime
typedef CUresult (*EncodeTiled2)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                 const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                 CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiled2 encoder() {
  static EncodeTiled2 fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult qr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &qr) == cudaSuccess &&
        qr == cudaDriverEntryPointSuccess)
      fn = (EncodeTiled2)p;
  }
  return fn;
}

souffle_status bert_init(Plan& p, void* ws, void* stream) {
  BertPlan& bp = p.bert;
  char* base = (char*)ws;
  auto ptr = [&](int node) -> char* { return (char*)p.buf_ptr[p.node_buf[node]]; };
  // packed constants: node -> copy in the workspace (snapshot of the bound values)
  std::vector<std::pair<int, int64_t>> packed;   // (node, byte offset)
  {
    int64_t off = bp.o_consts;
    for (const BertLayerIds& L : bp.layers)
      for (int nd : {L.bq, L.bk, L.bv, L.bo, L.g1, L.be1, L.c1, L.c2, L.g2, L.be2}) {
        packed.push_back({nd, off});
        off += 4 * numel(p.g.nodes[nd].shape);
      }
  }
  auto cptr = [&](int node) -> const float* {
    for (auto& q : packed)
      if (q.first == node) return (const float*)(base + q.second);
    return nullptr;
  };
  const int64_t S = bp.S, H = bp.H, F = bp.F;
  const int nl = (int)bp.layers.size();
  // ---- tensor maps (kActMaps activation maps, then per layer Wq Wk Wv Wo W1 W2)
  EncodeTiled2 enc = encoder();
  if (!enc) return fail(SOUFFLE_E_CUDA, "cuTensorMapEncodeTiled unavailable");
  std::vector<uint8_t> tm(128 * (kActMaps + 6 * (size_t)nl), 0);
  // bf16 tensor of `rank` dims (innermost first), row-major strides, 128B swizzle
  auto make = [&](int idx, void* gptr, int rank, std::vector<uint64_t> dims, std::vector<uint32_t> box) -> bool {
    CUtensorMap* m = (CUtensorMap*)&tm[128 * (size_t)idx];
    cuuint64_t d[3], st[2];
    cuuint32_t bx[3], es[3] = {1, 1, 1};
    uint64_t stride = 2;
    for (int i = 0; i < rank; ++i) {
      d[i] = dims[i];
      bx[i] = box[i];
      if (i > 0) st[i - 1] = stride;
      stride *= dims[i];
    }
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, rank, gptr, d, st, bx, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
  };
  auto m2 = [&](int idx, void* gptr, int64_t rows, int64_t cols, int box_rows) {
    return make(idx, gptr, 2, {(uint64_t)cols, (uint64_t)rows}, {64u, (uint32_t)box_rows});
  };
  bool ok = m2(MAP_XB, base + bp.o_xb, S, H, 128) && m2(MAP_CTX, base + bp.o_ctx, S, H, 128) &&
            m2(MAP_L1B, base + bp.o_l1b, S, H, 128) && m2(MAP_H, base + bp.o_h, S, F, 128) &&
            make(MAP_QK, base + bp.o_qk, 3, {64, (uint64_t)S, 2 * (uint64_t)bp.heads}, {64, 128, 1}) &&
            make(MAP_VT, base + bp.o_vt, 3, {(uint64_t)S, 64, (uint64_t)bp.heads}, {64, 64, 1});
  for (int l = 0; l < nl && ok; ++l) {
    const BertLayerIds& L = bp.layers[l];
    const int t = kActMaps + 6 * l;
    ok = m2(t + 0, ptr(L.Wq), H, H, bp.qkv.nt) && m2(t + 1, ptr(L.Wk), H, H, bp.qkv.nt) &&
         m2(t + 2, ptr(L.Wv), H, H, bp.qkv.nt) && m2(t + 3, ptr(L.Wo), H, H, bp.out.nt) &&
         m2(t + 4, ptr(L.W1), F, H, bp.ffn1.nt) && m2(t + 5, ptr(L.W2), H, F, bp.ffn2.nt);
  }
  if (!ok) return fail(SOUFFLE_E_CUDA, "cuTensorMapEncodeTiled failed (pointer alignment?)");
  // ---- stage table
  float* l1f = (float*)(base + bp.o_l1f);
  float* xf = (float*)(base + bp.o_xf);
  float* part_o = (float*)(base + bp.o_part_o);
  float* part_2 = (float*)(base + bp.o_part_2);
  uint16_t* xb = (uint16_t*)(base + bp.o_xb);
  uint16_t* l1b = (uint16_t*)(base + bp.o_l1b);
  uint16_t* ctx = (uint16_t*)(base + bp.o_ctx);
  uint16_t* hb = (uint16_t*)(base + bp.o_h);
  uint16_t* qk = (uint16_t*)(base + bp.o_qk);
  uint16_t* vt = (uint16_t*)(base + bp.o_vt);
  const float* X = (const float*)ptr(bp.X);
  float* Y = (float*)ptr(bp.Y);
  unsigned* ctrl = (unsigned*)(base + bp.o_ctrl);
  // point-to-point flags instead of the grid barriers QKV -> attention (head h reads only the Q/K/V tiles
  // of head h) and FFN1 -> FFN2 (K split s reads only the FFN1 tiles of its K range).  Opt-in
  // (SOUFFLE_BERT_P2P=1): measured on B200 the producer's release (fence + red, ~1 us after its
  // stores) plus the consumer's acquire poll costs as much as the 148-CTA barrier, because all
  // producers of a stage finish within ~0.2 us of each other.
  const bool nop2p = std::getenv("SOUFFLE_BERT_P2P") == nullptr;
  const bool p2p_qkv = !nop2p && bp.d % bp.qkv.nt == 0;
  const bool p2p_ffn = !nop2p && (bp.ffn2.kchunks * 64) % bp.ffn1.nt == 0 && F % (bp.ffn2.kchunks * 64) == 0;
  std::vector<BStage> st;
  auto stage = [&](int kind, int layer) {
    BStage s;
    std::memset(&s, 0, sizeof(s));
    s.kind = kind;
    s.layer = layer;
    return s;
  };
  auto gemm = [&](int layer, const BertGemmCfg& c, int64_t N, int64_t K, int wmap0, int64_t wrows, int amap, int epi) {
    BStage s = stage(BS_GEMM, layer);
    s.nt = c.nt; s.tiles_n = c.tiles_n; s.nsplit = c.nsplit; s.kchunks = c.kchunks;
    s.ntasks = c.tiles_n * c.nsplit;
    s.K = (int)K; s.N = (int)N; s.wmap0 = wmap0; s.wrows = (int)wrows;
    s.amap = amap; s.epi = epi; s.heads = bp.heads;
    return s;
  };
  auto ln = [&](int layer, const float* part, int nsplit, const float* bias, const float* res, const float* g,
                const float* b, float* out_f, uint16_t* out_b) {
    BStage s = stage(BS_ROW, layer);
    s.row_mode = 1; s.cols = (int)H; s.eps = (float)bp.eps; s.ntasks = (int)S;
    s.r_in = part; s.r_nsplit = nsplit; s.r_bias = bias; s.r_res = res; s.r_gamma = g; s.r_beta = b;
    s.r_out_f = out_f; s.r_out_b = out_b;
    return s;
  };
  {
    BStage s = stage(BS_ROW, -1);
    s.row_mode = 0; s.cols = (int)H; s.r_in = X; s.r_out_b = xb;
    s.ntasks = (int)S;
    st.push_back(s);
  }
  for (int l = 0; l < nl; ++l) {
    const BertLayerIds& L = bp.layers[l];
    const int t = kActMaps + 6 * l;
    const float* xin = l == 0 ? X : xf;
    BStage a = gemm(l, bp.qkv, 3 * H, H, t + 0, H, MAP_XB, EP_QKV);
    a.cpair = bp.pairs ? 1 : 0;
    a.bias = cptr(L.bq);   // bq, bk, bv are packed contiguously: the [Q | K | V] bias
    a.out_b = qk; a.out_vt = vt;
    st.push_back(a);
    unsigned* fl_qkv = ctrl + bp.nstages + 1 + 32 * (l * (bp.heads + bp.ffn2.nsplit));
    unsigned* fl_ffn = fl_qkv + 32 * bp.heads;
    if (p2p_qkv) { st.back().fout = fl_qkv; st.back().fdiv = bp.d; st.back().fmod = (int)H; }   // the QKV stage
    BStage at = stage(BS_ATTN, l);
    if (p2p_qkv) { at.fwait = 1; at.fin = fl_qkv; at.fneed = 3 * (bp.d / bp.qkv.nt); }
    at.heads = bp.heads; at.d = bp.d; at.H = (int)H;
    at.qkmap = MAP_QK; at.vtmap = MAP_VT;
    at.scale = (float)(1.0 / std::sqrt((double)bp.d));
    at.nt = bp.out.nt; at.tiles_n = bp.out.tiles_n; at.nsplit = bp.heads; at.kchunks = 1;
    at.ntasks = bp.out.tiles_n * bp.heads;
    at.K = (int)H; at.N = (int)H; at.wmap0 = t + 3; at.wrows = (int)H;
    at.epi = EP_PARTIAL; at.part = part_o;
    st.push_back(at);
    st.push_back(ln(l, part_o, bp.out.nsplit, cptr(L.bo), xin, cptr(L.g1), cptr(L.be1), l1f, l1b));
    BStage f1 = gemm(l, bp.ffn1, F, H, t + 4, F, MAP_L1B, EP_GELU);
    f1.cpair = bp.pairs ? 1 : 0;
    f1.bias = cptr(L.c1); f1.out_b = hb;
    if (p2p_ffn) { f1.fout = fl_ffn; f1.fdiv = bp.ffn2.kchunks * 64; f1.fmod = (int)F; }
    st.push_back(f1);
    BStage f2 = gemm(l, bp.ffn2, H, F, t + 5, H, MAP_H, EP_PARTIAL);
    f2.part = part_2;
    if (p2p_ffn) { f2.fwait = 1; f2.fin = fl_ffn; f2.fneed = bp.ffn2.kchunks * 64 / bp.ffn1.nt; }
    st.push_back(f2);
    const bool last = l == nl - 1;
    st.push_back(ln(l, part_2, bp.ffn2.nsplit, cptr(L.c2), l1f, cptr(L.g2), cptr(L.be2), last ? Y : xf,
                    last ? nullptr : xb));
  }
  if ((int)st.size() != bp.nstages) return fail(SOUFFLE_E_STATE, "internal: stage count");
  for (int i = 0; i < (int)st.size(); ++i) {
    st[i].idx = i;
    // barrier arrivals = CTAs with work (must match has_work() in kernels/bert.cu); stage 0 (convert +
    // constant refresh) runs on every CTA
    st[i].workers = st[i].kind == BS_ROW ? (st[i].row_mode == 0 ? bp.num_sms : std::min(bp.S, bp.num_sms))
                                         : st[i].ntasks;
  }
  for (int i = 0; i + 1 < (int)st.size(); ++i) st[i].arrive = st[i + 1].fwait ? 0 : 1;
  cudaStream_t s = (cudaStream_t)stream;
  cudaError_t e = cudaMemsetAsync(base, 0, (size_t)bp.total, s);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(base + bp.o_stages, st.data(), st.size() * sizeof(BStage), cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(base + bp.o_tmaps, tm.data(), tm.size(), cudaMemcpyHostToDevice, s);
  // constant vectors: copied from the bound pointers by stage 0 of every launch (BCopy table)
  std::vector<BCopy> cp;
  int total = 0;
  for (auto& q : packed) {
    BCopy c;
    c.src = (const float*)ptr(q.first);
    c.dst = (float*)(base + q.second);
    c.n = (int)numel(p.g.nodes[q.first].shape);
    c.first = total;
    total += c.n;
    cp.push_back(c);
  }
  bp.ncopies = (int)cp.size();
  bp.copy_total = total;
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(base + bp.o_copies, cp.data(), cp.size() * sizeof(BCopy), cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);   // host staging vectors die with this call
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("bert workspace init: ") + cudaGetErrorString(e));
  p.inited_ws = ws;
  p.dirty = false;
  return SOUFFLE_OK;
}

souffle_status bert_run(Plan& p, void* ws, void* stream) {
  BertPlan& bp = p.bert;
  static int max_active = -1;
  if (max_active < 0) {
    int b = 0;
    cudaError_t e = bert_max_active(&b);
    if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("occupancy query: ") + cudaGetErrorString(e));
    max_active = b;
  }
  int dev = 0, nsm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const int grid = bp.num_sms;   // the stage table's barrier arrival counts assume this grid
  if (nsm < grid) return fail(SOUFFLE_E_RESOURCE, "plan was built for " + std::to_string(grid) + " SMs");
  int need = 0;
  for (const BertGemmCfg* q : {&bp.qkv, &bp.out, &bp.ffn1, &bp.ffn2}) need = std::max(need, q->tiles_n * q->nsplit);
  need = std::max(need, bp.heads);
  if (max_active < 1 || grid < need)
    return fail(SOUFFLE_E_RESOURCE, "BERT persistent kernel needs " + std::to_string(need) + " co-resident CTAs");
  if (bp.pairs) {   // every CTA pair must be co-resident (the launch is not cooperative, see bert_launch)
    static int max_clusters = -1;
    if (max_clusters < 0) {
      int c = 0;
      cudaError_t e = bert_max_clusters(grid, &c);
      if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("cluster occupancy query: ") + cudaGetErrorString(e));
      max_clusters = c;
    }
    if (max_clusters * 2 < grid)
      return fail(SOUFFLE_E_RESOURCE, "only " + std::to_string(max_clusters) + " CTA pairs can be co-resident, need " +
                                          std::to_string(grid / 2));
  }
  char* base = (char*)ws;
  BertParams prm;
  std::memset(&prm, 0, sizeof(prm));
  prm.stages = (const BStage*)(base + bp.o_stages);
  prm.tmaps = base + bp.o_tmaps;
  prm.ctrl = (unsigned*)(base + bp.o_ctrl);
  prm.prof = p.profiling ? (unsigned long long*)(base + bp.o_prof) : nullptr;
  prm.nstages = bp.nstages;
  prm.nflags = bp.nflags;
  prm.S = bp.S;
  prm.copies = (const BCopy*)(base + bp.o_copies);
  prm.ncopies = bp.ncopies;
  prm.copy_total = bp.copy_total;
  if (const char* dbg = std::getenv("SOUFFLE_BERT_DBG_SKIP")) prm.dbg_skip = std::atoi(dbg);   // timing studies
  prm.s_begin = 0;
  prm.s_end = bp.nstages;
  prm.pairs = bp.pairs ? 1 : 0;
  // stage-isolation tests (tests/test_gpu_bert_stages.py): run only stages [b, e) on a workspace the
  // test pre-filled (the integer bit-exact checks of single GEMM stages)
  if (const char* se = std::getenv("SOUFFLE_BERT_STAGES")) {
    int b = 0, en = 0;
    if (std::sscanf(se, "%d,%d", &b, &en) == 2 && 0 <= b && b < en && en <= bp.nstages) {
      prm.s_begin = b;
      prm.s_end = en;
    }
  }
  cudaError_t e = bert_launch(prm, grid, bp.pairs, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("bert launch: ") + cudaGetErrorString(e));
  return SOUFFLE_OK;
}

}  // namespace souffle
