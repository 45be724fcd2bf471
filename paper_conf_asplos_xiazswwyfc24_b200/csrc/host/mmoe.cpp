// MMoE pattern: strict match of models.mmoe's TE program and launch of the fused kernel
// (kernels/mmoe.cu).  PAPER.md Table 2, §6.1 (horizontal fusion of the expert and gate GEMMs),
// Table 5 (one kernel).
#include <cstdlib>
#include <cstring>
#include <array>
#include <sstream>
#include <vector>
#include <string>

#include <cuda_runtime.h>

#include "../mmoe_types.h"
#include "plan.h"

namespace souffle {

souffle_status fail(souffle_status c, const std::string& m);
cudaError_t mmoe_launch(const MmoeParams& prm, cudaStream_t s);
size_t mmoe_smem_bytes(int B, int D, int E, int De, int T, int Th);
bool mmoe_cluster_ok(int B, int D, int E, int De, int T);

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
  int ph(std::vector<int64_t> shape, int dtype) {
    const Node* n = take(SOUFFLE_OP_PLACEHOLDER);
    if (!n || !n->is_const || n->shape != shape || n->dtype != dtype) { ok = false; return -1; }
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
  int red(int fn, int in) {
    const Node* n = take(SOUFFLE_OP_REDUCE);
    if (!n || n->fn != fn || n->in[0] != in || n->axis != 1 || !n->keepdim) { ok = false; return -1; }
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
}  // namespace

void mmoe_match(const Graph& g, const Analysis& an, uint32_t flags, MmoePlan& mp) {
  mp = MmoePlan();
  auto no = [&](const char* why) { mp.on = false; mp.why_not = why; };
  if (flags != 0) return no("ablation flags select the generic executor");
  const auto& N = g.nodes;
  if (N.size() < 6 || N[0].op != SOUFFLE_OP_PLACEHOLDER || N[0].is_const || N[0].shape.size() != 2 ||
      N[0].dtype != SOUFFLE_F32 || N[1].op != SOUFFLE_OP_PLACEHOLDER || N[1].shape.size() != 2)
    return no("not an MMoE program");
  mp.x = 0;
  mp.B = (int)N[0].shape[0];
  mp.D = (int)N[0].shape[1];
  mp.De = (int)N[1].shape[0];
  const int wd = N[1].dtype;
  mp.w_f32 = wd == SOUFFLE_F32;
  const int64_t B = mp.B, D = mp.D, De = mp.De;
  Cur c(g);
  c.i = 1;
  std::vector<int> ex, xmm;   // xmm: the expert and gate matmuls (all read x)
  // experts: until the first placeholder whose row count differs from De (the first gate)
  while (c.ok && c.i < N.size() && N[c.i].op == SOUFFLE_OP_PLACEHOLDER && N[c.i].shape.size() == 2 &&
         N[c.i].shape[0] == De && N[c.i].shape[1] == D) {
    mp.We.push_back(c.ph({De, D}, wd));
    int m = c.mm(mp.x, mp.We.back());
    xmm.push_back(m);
    mp.be.push_back(c.ph({De}, SOUFFLE_F32));
    ex.push_back(c.ew(SOUFFLE_EW_RELU, {c.ew(SOUFFLE_EW_ADD, {m, mp.be.back()})}));
  }
  mp.E = (int)mp.We.size();
  const int64_t E = mp.E;
  std::vector<int> gates;
  while (c.ok && c.i < N.size() && N[c.i].op == SOUFFLE_OP_PLACEHOLDER && N[c.i].shape.size() == 2 &&
         N[c.i].shape[0] == E && N[c.i].shape[1] == D) {
    mp.Wg.push_back(c.ph({E, D}, wd));
    int m = c.mm(mp.x, mp.Wg.back());
    xmm.push_back(m);
    mp.bg.push_back(c.ph({E}, SOUFFLE_F32));
    int a = c.ew(SOUFFLE_EW_ADD, {m, mp.bg.back()});
    int mx = c.red(SOUFFLE_RED_MAX, a);
    int ee = c.ew(SOUFFLE_EW_EXP, {c.ew(SOUFFLE_EW_SUB, {a, mx})});
    int z = c.red(SOUFFLE_RED_SUM, ee);
    gates.push_back(c.ew(SOUFFLE_EW_DIV, {ee, z}));
  }
  mp.T = (int)gates.size();
  if (!c.ok || mp.E < 1 || mp.T < 1) return no("not an MMoE program (experts / gates)");
  for (int k = 0; k < mp.T && c.ok; ++k) {
    int acc = -1;
    for (int e = 0; e < mp.E && c.ok; ++e) {
      int s = c.slice(gates[k], {0, e}, {B, e + 1});
      int p = c.ew(SOUFFLE_EW_MUL, {s, ex[e]});
      acc = acc < 0 ? p : c.ew(SOUFFLE_EW_ADD, {acc, p});
    }
    if (!c.ok || c.i >= N.size() || N[c.i].shape.size() != 2) { c.ok = false; break; }
    if (k == 0) mp.Th = (int)N[c.i].shape[0];
    const int64_t Th = mp.Th;
    mp.Wt.push_back(c.ph({Th, De}, wd));
    int t0 = c.mm(acc, mp.Wt.back());
    mp.bt.push_back(c.ph({Th}, SOUFFLE_F32));
    int t2 = c.ew(SOUFFLE_EW_RELU, {c.ew(SOUFFLE_EW_ADD, {t0, mp.bt.back()})});
    mp.Wo.push_back(c.ph({1, Th}, wd));
    int y0 = c.mm(t2, mp.Wo.back());
    mp.bo.push_back(c.ph({1}, SOUFFLE_F32));
    mp.y.push_back(c.ew(SOUFFLE_EW_ADD, {y0, mp.bo.back()}));
  }
  if (!c.ok || c.i != N.size()) return no("not an MMoE program (towers)");
  if (g.outputs != mp.y) return no("outputs are not the task towers");
  if (an.num_sp != 1) return no("the partition has more than one subprogram");
  for (size_t i = 0; i < g.nodes.size(); ++i)
    if (g.nodes[i].op != SOUFFLE_OP_PLACEHOLDER && an.assign[i] != 0) return no("TE outside subprogram 0");
  {
    const int gid = xmm.empty() || xmm[0] < 0 ? -1 : an.hgid[xmm[0]];
    bool one = gid >= 0 && an.hkind[gid] == 0;
    for (int m : xmm) one = one && m >= 0 && an.hgid[m] == gid;
    if (!one) return no("the analysis did not group the expert and gate matmuls into one N-concat GEMM (§6.1)");
  }
  if (mp.E > MMOE_MAX_E || mp.T > MMOE_MAX_T || mp.B > MMOE_MAX_B) return no("too many experts / tasks / rows");
  if (mp.B * mp.T > MMOE_THREADS / 32 || mp.Th > 32) return no("batch x tasks > warps or tower width > 32");
  if (1 + mp.E + 3 * mp.T > 32) return no("more than 32 parameter segments (one warp builds the staging table)");
  {   // parameter staging (kernels/mmoe.cu): <= 4 x 1024 16-byte weight units, <= 1024 vector elements
    const int64_t es2 = mp.w_f32 ? 4 : 2;
    const int64_t w16 = ((int64_t)mp.E * mp.De * mp.D + (int64_t)mp.T * (mp.E * mp.D + mp.Th * mp.De + mp.Th)) * es2 / 16;
    const int64_t vec = (int64_t)mp.B * mp.D + (int64_t)mp.E * mp.De + (int64_t)mp.T * (mp.E + mp.Th + 1);
    if (w16 > 4 * MMOE_THREADS || vec > MMOE_THREADS) return no("parameters exceed the staging capacity");
  }
  const int epv = mp.w_f32 ? 4 : 8;   // weight tensors are staged by bulk copies of 16-byte multiples
  if ((int64_t)mp.De * mp.D % epv || (int64_t)mp.E * mp.D % epv || (int64_t)mp.Th * mp.De % epv || mp.Th % epv)
    return no("weight tensor sizes must be multiples of 16 bytes");
  if (mmoe_smem_bytes(mp.B, mp.D, mp.E, mp.De, mp.T, mp.Th) > (size_t)MMOE_MAX_SMEM)
    return no("parameters do not fit one CTA's shared memory");
  mp.on = true;
}

std::string mmoe_describe(const MmoePlan& mp) {
  std::ostringstream os;
  if (!mp.on) {
    os << "pattern mmoe: not used (" << mp.why_not << ")\n";
    return os.str();
  }
  os << "pattern mmoe: " << mp.E << " experts x " << mp.De << ", " << mp.T << " tasks, d_in " << mp.D << ", batch "
     << mp.B << " -> 1 launch (kernels/mmoe.cu): horizontally fused expert+gate GEMM, softmax gates, mixture and towers";
  if (mmoe_cluster_ok(mp.B, mp.D, mp.E, mp.De, mp.T))
    os << "; cluster of " << MMOE_CL << " CTAs: the fused GEMM split by rows (weights streamed from global memory, "
          "results to CTA 0 over DSMEM), the rest in CTA 0\n";
  else
    os << " in one CTA, parameters staged once in shared memory\n";
  return os.str();
}

// parameter staging table (kernels/mmoe.cu): the shared-memory layout of the kernel, the bound
// pointers and the unit prefix sums, uploaded once per workspace initialisation
souffle_status mmoe_init(Plan& p, void* ws, void* stream) {
  const MmoePlan& mp = p.mmoe;
  auto ptr = [&](int node) -> uint64_t { return (uint64_t)(uintptr_t)p.buf_ptr[p.node_buf[node]]; };
  const int64_t es = mp.w_f32 ? 4 : 2, B = mp.B, D = mp.D, E = mp.E, De = mp.De, T = mp.T, Th = mp.Th;
  const int64_t R = E * De + T * E;
  auto a16 = [](int64_t x) { return (x + 15) & ~int64_t(15); };
  const int64_t oW1 = 0, oWt = a16(R * D * es), oWo = oWt + a16(T * Th * De * es), oxs = oWo + a16(T * Th * es);
  const int64_t ob1 = oxs + 4 * B * D, obt = ob1 + 4 * R, obo = obt + 4 * T * Th;
  std::vector<uint32_t> tab(2 * MMOE_SEG * 4, 0u);
  int nseg[2] = {0, 0};
  for (int t = 0; t < 2; ++t) {
    std::vector<std::array<int64_t, 3>> segs;   // (src, smem offset, units)
    if (t == 0) {
      for (int e = 0; e < E; ++e) segs.push_back({(int64_t)ptr(mp.We[e]), oW1 + e * De * D * es, De * D * es / 16});
      for (int k = 0; k < T; ++k) {
        segs.push_back({(int64_t)ptr(mp.Wg[k]), oW1 + (E * De + k * E) * D * es, E * D * es / 16});
        segs.push_back({(int64_t)ptr(mp.Wt[k]), oWt + k * Th * De * es, Th * De * es / 16});
        segs.push_back({(int64_t)ptr(mp.Wo[k]), oWo + k * Th * es, Th * es / 16});
      }
    } else {
      segs.push_back({(int64_t)ptr(mp.x), oxs, B * D});
      for (int e = 0; e < E; ++e) segs.push_back({(int64_t)ptr(mp.be[e]), ob1 + 4 * e * De, De});
      for (int k = 0; k < T; ++k) {
        segs.push_back({(int64_t)ptr(mp.bg[k]), ob1 + 4 * (E * De + k * E), E});
        segs.push_back({(int64_t)ptr(mp.bt[k]), obt + 4 * k * Th, Th});
        segs.push_back({(int64_t)ptr(mp.bo[k]), obo + 4 * k, 1});
      }
    }
    if ((int)segs.size() + 1 > MMOE_SEG) return fail(SOUFFLE_E_UNSUPPORTED, "MMoE staging table overflow");
    int64_t pre = 0;
    for (size_t j = 0; j <= segs.size(); ++j) {
      uint32_t* e = &tab[(t * MMOE_SEG + j) * 4];
      const uint64_t src = j < segs.size() ? (uint64_t)segs[j][0] : 0;
      e[0] = (uint32_t)src;
      e[1] = (uint32_t)(src >> 32);
      e[2] = j < segs.size() ? (uint32_t)segs[j][1] : 0u;
      e[3] = (uint32_t)pre;
      if (j < segs.size()) pre += segs[j][2];
    }
    nseg[t] = (int)segs.size();
  }
  p.mmoe.nseg[0] = nseg[0];
  p.mmoe.nseg[1] = nseg[1];
  cudaError_t e = cudaMemcpyAsync(ws, tab.data(), tab.size() * 4, cudaMemcpyHostToDevice, (cudaStream_t)stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize((cudaStream_t)stream);   // the host table is a local
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("mmoe workspace init: ") + cudaGetErrorString(e));
  p.inited_ws = ws;
  p.dirty = false;
  return SOUFFLE_OK;
}

souffle_status mmoe_run(Plan& p, void* ws, void* stream) {
  MmoePlan& mp = p.mmoe;
  auto ptr = [&](int node) -> void* { return p.buf_ptr[p.node_buf[node]]; };
  MmoeParams prm;
  std::memset(&prm, 0, sizeof(prm));
  prm.x = (const float*)ptr(mp.x);
  for (int e = 0; e < mp.E; ++e) {
    prm.We[e] = ptr(mp.We[e]);
    prm.be[e] = (const float*)ptr(mp.be[e]);
  }
  for (int k = 0; k < mp.T; ++k) {
    prm.Wg[k] = ptr(mp.Wg[k]);
    prm.bg[k] = (const float*)ptr(mp.bg[k]);
    prm.Wt[k] = ptr(mp.Wt[k]);
    prm.bt[k] = (const float*)ptr(mp.bt[k]);
    prm.Wo[k] = ptr(mp.Wo[k]);
    prm.bo[k] = (const float*)ptr(mp.bo[k]);
    prm.y[k] = (float*)ptr(mp.y[k]);
  }
  prm.B = mp.B; prm.D = mp.D; prm.E = mp.E; prm.De = mp.De; prm.T = mp.T; prm.Th = mp.Th;
  prm.w_f32 = mp.w_f32;
  prm.pad = std::getenv("SOUFFLE_MMOE_DEBUG") ? 1 : 0;   // debug: per-phase clock deltas (printf)
  prm.seg = (const uint4*)ws;
  prm.nseg[0] = mp.nseg[0];
  prm.nseg[1] = mp.nseg[1];
  for (int k = 0; k < mp.E; ++k)
    if ((uintptr_t)prm.We[k] & 15) return fail(SOUFFLE_E_INVALID_ARG, "MMoE weights must be 16-byte aligned");
  for (int k = 0; k < mp.T; ++k)
    if (((uintptr_t)prm.Wg[k] | (uintptr_t)prm.Wt[k] | (uintptr_t)prm.Wo[k]) & 15)
      return fail(SOUFFLE_E_INVALID_ARG, "MMoE weights must be 16-byte aligned");
  cudaError_t e = mmoe_launch(prm, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("mmoe launch: ") + cudaGetErrorString(e));
  return SOUFFLE_OK;
}

}  // namespace souffle
