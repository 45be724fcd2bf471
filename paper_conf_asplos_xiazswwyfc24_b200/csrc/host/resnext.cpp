// ResNeXt Bottleneck pattern (Table 2, ResNeXt-101 64 x 4d): strict TE match of the block's
// program (models.resnext), workspace layout and launch of kernels/resnext.cu.
#include <cmath>
#include <cstdlib>
#include <sstream>
#include <string>

#include <cuda_runtime.h>

#include "plan.h"
#include "resnext.h"

namespace souffle {

souffle_status fail(souffle_status c, const std::string& m);
cudaError_t resnext_launch(const RxParams& prm, int grid, cudaStream_t s);

namespace {
int64_t al(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

// sequential matcher over the node list (the builder emits a fixed order)
struct Cur {
  const Graph& g;
  size_t i = 0;
  bool ok = true;
  explicit Cur(const Graph& gr) : g(gr) {}
  const Node* peek() const { return i < g.nodes.size() ? &g.nodes[i] : nullptr; }
  const Node* take(int op) {
    if (!ok || i >= g.nodes.size() || g.nodes[i].op != op) { ok = false; return nullptr; }
    return &g.nodes[i++];
  }
  int id() const { return (int)i - 1; }
  int ph(std::vector<int64_t> shape, int is_const = 1) {
    const Node* n = take(SOUFFLE_OP_PLACEHOLDER);
    if (!n || n->shape != shape || n->dtype != SOUFFLE_F32 || n->is_const != is_const) { ok = false; return -1; }
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
  int reshape(int in, std::vector<int64_t> shape) {
    const Node* n = take(SOUFFLE_OP_RESHAPE);
    if (!n || n->in[0] != in || n->shape != shape) { ok = false; return -1; }
    return id();
  }
  int permute(int in, std::vector<int> perm) {
    const Node* n = take(SOUFFLE_OP_PERMUTE);
    if (!n || n->in[0] != in || n->perm != perm) { ok = false; return -1; }
    return id();
  }
  int slice2(int in, int64_t H, int64_t C) {   // [::2, ::2, :] of an [H, H, C] tensor
    const Node* n = take(SOUFFLE_OP_SLICE);
    if (!n || n->in[0] != in || n->begin != std::vector<int64_t>{0, 0, 0} || n->end != std::vector<int64_t>{H, H, C} ||
        n->stride != std::vector<int64_t>{2, 2, 1}) { ok = false; return -1; }
    return id();
  }
  // BN (per-channel scale, bias): mul(v, s), add(., b)
  int bn(int v, int64_t C, int* s, int* b) {
    *s = ph({C});
    *b = ph({C});
    return ew(SOUFFLE_EW_ADD, {ew(SOUFFLE_EW_MUL, {v, *s}), *b});
  }
};
}  // namespace

void resnext_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, RxPlan& rp) {
  rp = RxPlan();
  for (int t = 0; t < RX_TAPS; ++t) rp.W2[t] = rp.m[t] = -1;
  auto no = [&](const char* why) { rp.on = false; rp.why_not = why; };
  if (flags != 0) return no("ablation flags select the generic executor");
  const auto& N = g.nodes;
  if (N.size() < 60 || N[0].op != SOUFFLE_OP_PLACEHOLDER || N[0].shape.size() != 2 || N[0].is_const ||
      N[0].dtype != SOUFFLE_F32 || N[1].op != SOUFFLE_OP_PLACEHOLDER || N[1].shape.size() != 2)
    return no("not a ResNeXt block");
  const int64_t HW = N[0].shape[0], cin = N[0].shape[1], w = N[1].shape[0];
  const int64_t H = (int64_t)std::llround(std::sqrt((double)HW));
  if (H * H != HW || H < 2) return no("input is not a square image");
  Cur c(g);
  rp.x = c.ph({HW, cin}, 0);
  rp.W1 = c.ph({w, cin});
  int a = c.bn(c.mm(rp.x, rp.W1), w, &rp.s1, &rp.b1);
  a = c.ew(SOUFFLE_EW_RELU, {a});
  const int a3 = c.reshape(a, {H, H, w});
  if (!c.ok) return no("not a ResNeXt block (1x1 convolution)");
  // grouped 3x3 taps: the first tap's grouping reshape gives (G, cg)
  int64_t G = 0, cg = 0;
  int acc = -1;
  for (int t = 0; t < RX_TAPS && c.ok; ++t) {
    const int i = t / 3, j = t % 3;
    int term = a3;
    if (!(i == 1 && j == 1)) {
      const Node* r = c.take(SOUFFLE_OP_ROLL);
      const std::vector<int64_t> want{((1 - i) % H + H) % H, ((1 - j) % H + H) % H, 0};
      if (!r || r->in[0] != a3 || r->shifts != want) return no("grouped-convolution tap roll");
      const int rid = c.id();
      rp.m[t] = c.ph({H, H, 1});
      term = c.ew(SOUFFLE_EW_MUL, {rid, rp.m[t]});
    }
    if (t == 0) {
      const Node* rs = c.peek();
      if (!rs || rs->op != SOUFFLE_OP_RESHAPE || rs->shape.size() != 3 || rs->shape[0] != HW) return no("group reshape");
      G = rs->shape[1];
      cg = rs->shape[2];
      if (G * cg != w || cg % 4 || G < 1) return no("groups x channels per group");
    }
    const int tg = c.permute(c.reshape(term, {HW, G, cg}), {1, 0, 2});
    rp.W2[t] = c.ph({G, cg, cg});
    const int pt = c.mm(tg, rp.W2[t]);
    acc = acc < 0 ? pt : c.ew(SOUFFLE_EW_ADD, {acc, pt});
  }
  int c3 = c.reshape(c.permute(acc, {1, 0, 2}), {H, H, w});
  if (!c.ok) return no("not a ResNeXt block (grouped convolution)");
  int64_t stride = 1;
  if (c.peek() && c.peek()->op == SOUFFLE_OP_SLICE) {
    if (H % 2) return no("stride 2 needs an even image size");
    c3 = c.slice2(c3, H, w);
    stride = 2;
  }
  const int64_t Ho = H / stride;
  int d = c.bn(c.reshape(c3, {Ho * Ho, w}), w, &rp.s2, &rp.b2);
  d = c.ew(SOUFFLE_EW_RELU, {d});
  if (!c.peek() || c.peek()->op != SOUFFLE_OP_PLACEHOLDER || c.peek()->shape.size() != 2) return no("1x1 convolution 3");
  const int64_t cout = c.peek()->shape[0];
  rp.W3 = c.ph({cout, w});
  int y = c.bn(c.mm(d, rp.W3), cout, &rp.s3, &rp.b3);
  int sc = rp.x;
  if (stride != 1 || cin != cout) {
    int xs = rp.x;
    if (stride != 1) xs = c.reshape(c.slice2(c.reshape(rp.x, {H, H, cin}), H, cin), {Ho * Ho, cin});
    rp.Wd = c.ph({cout, cin});
    sc = c.bn(c.mm(xs, rp.Wd), cout, &rp.sd, &rp.bd);
  }
  y = c.ew(SOUFFLE_EW_RELU, {c.ew(SOUFFLE_EW_ADD, {y, sc})});
  if (!c.ok || c.i != N.size()) return no("not a ResNeXt block");
  if (cin % 16 || w % 16 || cout % 16) return no("channel counts must be multiples of 16 (vector GEMM slabs)");
  if (g.outputs.size() != 1 || g.outputs[0] != y) return no("the only output must be the block output");
  const int sms = dev.num_sms > 0 ? dev.num_sms : 148;
  rp.y = y;
  rp.H = (int)H; rp.cin = (int)cin; rp.w = (int)w; rp.G = (int)G; rp.stride = (int)stride; rp.cout = (int)cout;
  rp.grid = sms; rp.num_sp = an.num_sp;
  int64_t o = 0;
  rp.o_ctrl = o; o = al(o + 256, 256);
  rp.o_a = o; o = al(o + 4 * HW * w, 256);
  rp.o_d = o; o = al(o + 4 * Ho * Ho * w, 256);
  rp.o_acc1 = o; o = al(o + 4 * HW * w, 256);
  rp.o_acc2 = o; o = al(o + 4 * Ho * Ho * cout, 256);
  rp.o_acc3 = o; o = al(o + 4 * Ho * Ho * cout, 256);
  rp.o_cnt = o; o = al(o + 4 * 3 * RX_MAX_TILES, 256);
  rp.total = al(o, 4096);
  if ((HW + 63) / 64 * ((w + 63) / 64) > RX_MAX_TILES || (Ho * Ho + 63) / 64 * ((cout + 63) / 64) > RX_MAX_TILES)
    return no("too many 64 x 64 GEMM tiles for the split-K counters");
  rp.on = true;
}

std::string resnext_describe(const RxPlan& rp) {
  std::ostringstream os;
  if (!rp.on) {
    os << "pattern resnext: not used (" << rp.why_not << ")\n";
    return os.str();
  }
  os << "pattern resnext: " << rp.cin << " -> " << rp.w << " (" << rp.G << " groups x " << rp.w / rp.G << ") -> "
     << rp.cout << " channels, stride " << rp.stride << ", " << rp.H << "x" << rp.H
     << (rp.Wd >= 0 ? ", projection shortcut" : ", identity shortcut")
     << " -> 1 persistent launch (kernels/resnext.cu), " << rp.grid
     << " CTAs, 2 grid barriers (the partition's " << rp.num_sp << " subprogram(s) end at barriers of the launch)\n";
  return os.str();
}

souffle_status resnext_run(Plan& p, void* ws, void* stream) {
  const RxPlan& rp = p.rx;
  auto ptr = [&](int node) -> const float* { return node < 0 ? nullptr : (const float*)p.buf_ptr[p.node_buf[node]]; };
  char* base = (char*)ws;
  RxParams prm{};
  prm.x = ptr(rp.x); prm.W1 = ptr(rp.W1); prm.s1 = ptr(rp.s1); prm.b1 = ptr(rp.b1);
  for (int t = 0; t < RX_TAPS; ++t) {
    prm.W2[t] = ptr(rp.W2[t]);
    prm.m[t] = ptr(rp.m[t]);
  }
  prm.s2 = ptr(rp.s2); prm.b2 = ptr(rp.b2); prm.W3 = ptr(rp.W3); prm.s3 = ptr(rp.s3); prm.b3 = ptr(rp.b3);
  prm.Wd = ptr(rp.Wd); prm.sd = ptr(rp.sd); prm.bd = ptr(rp.bd);
  prm.y = (float*)p.buf_ptr[p.node_buf[rp.y]];
  prm.a = (float*)(base + rp.o_a);
  prm.d = (float*)(base + rp.o_d);
  prm.ctrl = (unsigned*)(base + rp.o_ctrl);
  prm.acc1 = (float*)(base + rp.o_acc1);
  prm.acc2 = (float*)(base + rp.o_acc2);
  prm.acc3 = (float*)(base + rp.o_acc3);
  prm.cnt = (unsigned*)(base + rp.o_cnt);
  if (std::getenv("SOUFFLE_RX_PROF")) prm.prof = (unsigned long long*)(base + rp.o_ctrl + 64);   // 4 stamps
  prm.H = rp.H; prm.cin = rp.cin; prm.w = rp.w; prm.G = rp.G; prm.stride = rp.stride; prm.cout = rp.cout;
  cudaError_t e = resnext_launch(prm, rp.grid, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("resnext launch: ") + cudaGetErrorString(e));
  return SOUFFLE_OK;
}

}  // namespace souffle
