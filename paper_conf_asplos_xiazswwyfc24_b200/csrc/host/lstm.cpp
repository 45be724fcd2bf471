// Stacked-LSTM pattern: strict match of the unrolled recurrence, layout, and launch of the
// persistent wavefront kernel (kernels/lstm.cu).  PAPER.md §8.4, Table 5 (one
// kernel), Table 6 (weights read once).
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <sstream>
#include <string>

#include <cuda_runtime.h>

#include "../lstm_types.h"
#include "plan.h"

namespace souffle {

extern thread_local std::string g_err;
souffle_status fail(souffle_status c, const std::string& m);
cudaError_t lstm_launch(const LstmParams& prm, int grid, cudaStream_t s);
size_t lstm_smem_bytes(int K_max, int w_f32);

namespace {

struct Cur {
  const Graph& g;
  size_t i = 0;
  bool ok = true;
  explicit Cur(const Graph& gr) : g(gr) {}
  const Node* take(int op) {
    if (!ok || i >= g.nodes.size() || g.nodes[i].op != op) { ok = false; return nullptr; }
    return &g.nodes[i++];
  }
  int id() const { return (int)i - 1; }
  int ph(std::vector<int64_t> shape, int dtype, int is_const) {
    const Node* n = take(SOUFFLE_OP_PLACEHOLDER);
    if (!n || n->shape != shape || n->dtype != dtype || n->is_const != is_const) { ok = false; return -1; }
    return id();
  }
  int mm(int a, int b) {
    const Node* n = take(SOUFFLE_OP_MATMUL);
    if (!n || n->a != a || n->b != b || !n->trans_b || n->prec != SOUFFLE_F32) { ok = false; return -1; }
    return id();
  }
  int ew(int fn, std::vector<int> in) {
    const Node* n = take(SOUFFLE_OP_ELEMENTWISE);
    if (!n || n->fn != fn || n->in != in) { ok = false; return -1; }
    return id();
  }
  int slice(int in, std::vector<int64_t> b, std::vector<int64_t> e) {
    const Node* n = take(SOUFFLE_OP_SLICE);
    if (!n || n->in[0] != in || n->begin != b || n->end != e || n->stride != std::vector<int64_t>{1, 1}) {
      ok = false;
      return -1;
    }
    return id();
  }
};

int64_t al(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

}  // namespace

void lstm_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, LstmPlan& lp) {
  lp = LstmPlan();
  auto no = [&](const char* why) { lp.on = false; lp.why_not = why; };
  if (flags != 0) return no("ablation flags select the generic executor");
  const auto& N = g.nodes;
  if (N.size() < 8 || N[0].op != SOUFFLE_OP_PLACEHOLDER || N[0].is_const || N[0].shape.size() != 2 ||
      N[0].dtype != SOUFFLE_F32)
    return no("first node is not an fp32 [T, I] input");
  lp.X = 0;
  lp.T = (int)N[0].shape[0];
  lp.I = (int)N[0].shape[1];
  if (N[1].op != SOUFFLE_OP_PLACEHOLDER || N[1].shape.size() != 2) return no("no W_ih");
  const int64_t H4 = N[1].shape[0];
  lp.H = (int)(H4 / 4);
  const int wd = N[1].dtype;
  lp.w_f32 = wd == SOUFFLE_F32;
  Cur c(g);
  c.i = 1;
  const int64_t H = lp.H;
  // per-layer placeholders until the first slice of X
  while (c.ok && c.i < N.size() && N[c.i].op == SOUFFLE_OP_PLACEHOLDER) {
    const int n = (int)lp.W.size();
    lp.W.push_back(c.ph({H4, n == 0 ? (int64_t)lp.I : H}, wd, 1));
    lp.U.push_back(c.ph({H4, H}, wd, 1));
    lp.bi.push_back(c.ph({H4}, SOUFFLE_F32, 1));
    lp.bh.push_back(c.ph({H4}, SOUFFLE_F32, 1));
    lp.h0.push_back(c.ph({1, H}, SOUFFLE_F32, 0));
    lp.c0.push_back(c.ph({1, H}, SOUFFLE_F32, 0));
  }
  lp.L = (int)lp.W.size();
  if (!c.ok || lp.L == 0) return no("placeholders are not LSTM layer parameters");
  std::vector<int> h(lp.h0), cc(lp.c0);
  for (int t = 0; t < lp.T && c.ok; ++t) {
    int x = c.slice(lp.X, {t, 0}, {t + 1, lp.I});
    for (int n = 0; n < lp.L && c.ok; ++n) {
      int g1 = c.ew(SOUFFLE_EW_ADD, {c.mm(x, lp.W[n]), lp.bi[n]});
      int m2 = c.mm(h[n], lp.U[n]);
      int g4 = c.ew(SOUFFLE_EW_ADD, {c.ew(SOUFFLE_EW_ADD, {g1, m2}), lp.bh[n]});
      int s[4];
      for (int k = 0; k < 4; ++k) s[k] = c.slice(g4, {0, k * H}, {1, (k + 1) * H});
      int i_ = c.ew(SOUFFLE_EW_SIGMOID, {s[0]});
      int f_ = c.ew(SOUFFLE_EW_SIGMOID, {s[1]});
      int g_ = c.ew(SOUFFLE_EW_TANH, {s[2]});
      int o_ = c.ew(SOUFFLE_EW_SIGMOID, {s[3]});
      int fc = c.ew(SOUFFLE_EW_MUL, {f_, cc[n]});
      int ig = c.ew(SOUFFLE_EW_MUL, {i_, g_});
      cc[n] = c.ew(SOUFFLE_EW_ADD, {fc, ig});
      int tc = c.ew(SOUFFLE_EW_TANH, {cc[n]});
      h[n] = c.ew(SOUFFLE_EW_MUL, {o_, tc});
      x = h[n];
    }
    lp.top.push_back(x);
  }
  if (!c.ok || c.i != N.size()) return no("TE program is not an unrolled stacked LSTM");
  std::vector<int> expect;   // souffle_mark_output de-duplicates (top[T-1] is h_n of the last layer)
  auto add = [&](int t) {
    if (std::find(expect.begin(), expect.end(), t) == expect.end()) expect.push_back(t);
  };
  for (int t : lp.top) add(t);
  for (int n = 0; n < lp.L; ++n) {
    add(h[n]);
    add(cc[n]);
  }
  if (g.outputs != expect) return no("outputs are not [top_t..., (h_n, c_n) per layer]");
  lp.hn = h;
  lp.cn = cc;
  if (an.num_sp != 1) return no("the partition has more than one subprogram");
  for (size_t i = 0; i < g.nodes.size(); ++i)
    if (g.nodes[i].op != SOUFFLE_OP_PLACEHOLDER && an.assign[i] != 0) return no("TE outside subprogram 0");
  // W_hh feeds the dependent chain h(t-1) -> h(t): temporal reuse; W_ih is spatial on layer 0 (its
  // inputs x_t are independent) and temporal above; either way the T GEMVs share the on-chip copy
  if (lp.T > 1)
    for (int n = 0; n < lp.L; ++n)
      if (an.reuse_kind[lp.W[n]] < 0 || an.reuse_kind[lp.U[n]] != 1)
        return no("the analysis found no reuse of a layer's weights across the steps (§5.1)");
  // ---- resources: NP CTAs per layer, each owning <= 32 hidden units (<= 128 gate rows) whose
  // weights stay resident in shared memory.  The per-step GEMV is bound by reading those weights
  // from shared memory, so NP is as large as the SMs allow (all layers' CTAs co-resident).
  if (lp.H % 8 || lp.I % 8) return no("needs H % 8 == 0 and I % 8 == 0");
  const int sms = dev.num_sms > 0 ? dev.num_sms : 148;
  const int np_min = (lp.H + LSTM_UNITS - 1) / LSTM_UNITS;
  lp.NP = std::max(np_min, std::min(sms / lp.L, lp.H / 8));
  // register-resident GEMV (K <= 512): the fewest CTAs per layer whose units fit the register layout
  // (<= 20 units) -- fewer producers per wavefront step to wait for (10 x 256: 13 CTAs per layer,
  // 170 vs 174 us at 14)
  {
    const char* fs = std::getenv("SOUFFLE_LSTM_SMEM");
    const int np_reg = std::max(np_min, (lp.H + LSTM_REG_UNITS - 1) / LSTM_REG_UNITS);
    if (std::max(lp.I, lp.H) + lp.H <= LSTM_REG_K && np_reg * lp.L <= sms && !(fs && std::atoi(fs))) lp.NP = np_reg;
  }
  if (const char* e = std::getenv("SOUFFLE_LSTM_NP")) {   // timing studies
    const int v = std::atoi(e);
    if (v >= np_min && v * lp.L <= sms && v <= lp.H) lp.NP = v;
  }
  lp.K_max = std::max(lp.I, lp.H) + lp.H;
  if (lp.K_max > 2 * LSTM_THREADS) return no("input + hidden width above 1024");
  if (lp.L * lp.NP > sms) return no("more CTAs than SMs");
  // weights in registers when a CTA's tile fits the register layout (K <= 512, <= 20 units);
  // SOUFFLE_LSTM_SMEM=1 forces the shared-memory kernel (A/B studies)
  const int nu_max = (lp.H + lp.NP - 1) / lp.NP;
  const char* force_smem = std::getenv("SOUFFLE_LSTM_SMEM");
  lp.reg = (lp.K_max <= LSTM_REG_K && nu_max <= LSTM_REG_UNITS && !(force_smem && std::atoi(force_smem))) ? 1 : 0;
  if (!lp.reg && lstm_smem_bytes(lp.K_max, lp.w_f32) > (size_t)LSTM_MAX_SMEM) return no("weights of 32 units do not fit shared memory");
  int64_t o = 0;
  lp.o_gen = o; o = al(o + 8, 256);
  lp.o_layers = o; o = al(o + (int64_t)sizeof(LstmLayer) * lp.L, 256);
  lp.o_top = o; o = al(o + 8 * (int64_t)lp.T, 256);
  lp.o_hbuf = o; o = al(o + 8 * (int64_t)lp.L * lp.T * lp.H, 256);
  lp.o_prof = o; o = al(o + 8 * 4 * (int64_t)lp.T, 256);
  lp.total = al(o, 4096);
  lp.on = true;
}

std::string lstm_describe(const LstmPlan& lp) {
  std::ostringstream os;
  if (!lp.on) {
    os << "pattern lstm: not used (" << lp.why_not << ")\n";
    return os.str();
  }
  os << "pattern lstm: " << lp.L << " layers x " << lp.T << " steps, H=" << lp.H << " I=" << lp.I << " ("
     << (lp.w_f32 ? "fp32" : "bf16") << " weights) -> 1 persistent launch (kernels/lstm.cu), " << lp.L * lp.NP
     << " CTAs = " << lp.NP << " per layer x <= " << (lp.H + lp.NP - 1) / lp.NP << " units, weights resident in "
     << (lp.reg ? "registers (fp32, packed FFMA2 GEMV)" : "shared memory") << ", wavefront of "
     << lp.L + lp.T - 1 << " dependent steps synchronised through tagged (value, step) words\n";
  return os.str();
}

souffle_status lstm_init(Plan& p, void* ws, void* stream) {
  LstmPlan& lp = p.lstm;
  char* base = (char*)ws;
  auto ptr = [&](int node) -> char* { return (char*)p.buf_ptr[p.node_buf[node]]; };
  std::vector<LstmLayer> layers(lp.L);
  for (int n = 0; n < lp.L; ++n) {
    LstmLayer& Ly = layers[n];
    std::memset(&Ly, 0, sizeof(Ly));
    Ly.W = ptr(lp.W[n]);
    Ly.U = ptr(lp.U[n]);
    Ly.b_ih = (const float*)ptr(lp.bi[n]);
    Ly.b_hh = (const float*)ptr(lp.bh[n]);
    Ly.h0 = (const float*)ptr(lp.h0[n]);
    Ly.c0 = (const float*)ptr(lp.c0[n]);
    Ly.h_n = (float*)ptr(lp.hn[n]);
    Ly.c_n = (float*)ptr(lp.cn[n]);
    Ly.in_dim = n == 0 ? lp.I : lp.H;
    for (const void* q : {Ly.W, Ly.U})
      if (((uintptr_t)q) & 15) return fail(SOUFFLE_E_INVALID_ARG, "LSTM weights must be 16-byte aligned");
  }
  std::vector<float*> top(lp.T);
  for (int t = 0; t < lp.T; ++t) top[t] = (float*)ptr(lp.top[t]);
  cudaStream_t s = (cudaStream_t)stream;
  cudaError_t e = cudaMemsetAsync(base, 0, (size_t)lp.total, s);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(base + lp.o_layers, layers.data(), layers.size() * sizeof(LstmLayer), cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(base + lp.o_top, top.data(), top.size() * sizeof(float*), cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("lstm workspace init: ") + cudaGetErrorString(e));
  p.inited_ws = ws;
  p.dirty = false;
  return SOUFFLE_OK;
}

souffle_status lstm_run(Plan& p, void* ws, void* stream) {
  LstmPlan& lp = p.lstm;
  char* base = (char*)ws;
  LstmParams prm;
  std::memset(&prm, 0, sizeof(prm));
  prm.layers = (const LstmLayer*)(base + lp.o_layers);
  prm.X = (const float*)p.buf_ptr[p.node_buf[lp.X]];
  prm.top = (float* const*)(base + lp.o_top);
  prm.hbuf = (uint2*)(base + lp.o_hbuf);
  prm.gen = (unsigned*)(base + lp.o_gen);
  prm.L = lp.L;
  prm.T = lp.T;
  prm.H = lp.H;
  prm.NP = lp.NP;
  prm.w_f32 = lp.w_f32;
  prm.K_max = lp.K_max;
  prm.reg = lp.reg;
  if (p.profiling) {   // debug timeline of one CTA (SOUFFLE_LSTM_PROF_CTA, default the middle layer)
    prm.prof = (unsigned long long*)(base + lp.o_prof);
    const char* e = std::getenv("SOUFFLE_LSTM_PROF_CTA");
    prm.prof_cta = e ? std::atoi(e) : (lp.L / 2) * lp.NP;
  }
  cudaError_t e = lstm_launch(prm, lp.L * lp.NP, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("lstm launch: ") + cudaGetErrorString(e));
  return SOUFFLE_OK;
}

}  // namespace souffle
