// EfficientNet MBConv pattern (Fig. 5 / 6): strict TE match of the block's program, workspace
// layout and launch of kernels/mbconv.cu.
#include <cmath>
#include <cstdlib>
#include <sstream>
#include <string>

#include <cuda_runtime.h>

#include "mbconv.h"
#include "plan.h"

namespace souffle {

souffle_status fail(souffle_status c, const std::string& m);
cudaError_t mbconv_launch(const MbParams& prm, int grid, cudaStream_t s);
size_t mbconv_reuse_smem(int pix_blk, int E, int cout);

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
  // BN (per-channel scale, bias) then optionally SiLU: mul(v, s), add(., b) [, sigmoid, mul]
  int bn(int v, int64_t C, int* s, int* b, bool act) {
    *s = ph({C});
    *b = ph({C});
    int r = ew(SOUFFLE_EW_ADD, {ew(SOUFFLE_EW_MUL, {v, *s}), *b});
    if (act) r = ew(SOUFFLE_EW_MUL, {r, ew(SOUFFLE_EW_SIGMOID, {r})});
    return r;
  }
};
}  // namespace

void mbconv_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, MbPlan& mp) {
  mp = MbPlan();
  for (int t = 0; t < MB_MAX_TAPS; ++t) mp.w[t] = mp.m[t] = -1;
  auto no = [&](const char* why) { mp.on = false; mp.why_not = why; };
  if (flags != 0 && flags != SOUFFLE_FLAG_NO_PREFETCH) return no("ablation flags select the generic executor");
  const auto& N = g.nodes;
  if (N.size() < 40 || N[0].op != SOUFFLE_OP_PLACEHOLDER || N[0].shape.size() != 2 || N[0].is_const ||
      N[0].dtype != SOUFFLE_F32)
    return no("not an MBConv program");
  const int64_t HW = N[0].shape[0], cin = N[0].shape[1];
  const int64_t H = (int64_t)std::llround(std::sqrt((double)HW));
  if (H * H != HW) return no("input is not a square image");
  Cur c(g);
  mp.x = c.ph({HW, cin}, 0);
  int a = mp.x;
  int64_t E = cin;
  if (c.peek() && c.peek()->op == SOUFFLE_OP_PLACEHOLDER) {   // 1x1 expand convolution
    const Node* we = c.peek();
    if (we->shape.size() != 2 || we->shape[1] != cin) return no("not an MBConv program");
    E = we->shape[0];
    mp.We = c.ph({E, cin});
    a = c.bn(c.mm(mp.x, mp.We), E, &mp.se, &mp.be, true);
  }
  const int a3 = c.reshape(a, {H, H, E});
  if (!c.ok) return no("not an MBConv program (expand)");
  // depthwise taps: the first tap's roll gives the padding (shift = pad - 0)
  if (!c.peek() || c.peek()->op != SOUFFLE_OP_ROLL || c.peek()->shifts.size() != 3) return no("no depthwise taps");
  const int64_t pad = c.peek()->shifts[0];
  const int64_t k = 2 * pad + 1;
  if (k < 3 || k * k > MB_MAX_TAPS || pad >= H) return no("depthwise kernel size");
  int acc = -1;
  for (int64_t t = 0; t < k * k && c.ok; ++t) {
    const int64_t i = t / k, j = t % k;
    int term = a3;
    if (!(i == pad && j == pad)) {
      const Node* r = c.take(SOUFFLE_OP_ROLL);
      const std::vector<int64_t> want{((pad - i) % H + H) % H, ((pad - j) % H + H) % H, 0};
      if (!r || r->in[0] != a3 || r->shifts != want) return no("depthwise tap roll");
      const int rid = c.id();
      mp.m[t] = c.ph({H, H, 1});
      term = c.ew(SOUFFLE_EW_MUL, {rid, mp.m[t]});
    }
    mp.w[t] = c.ph({E});
    term = c.ew(SOUFFLE_EW_MUL, {term, mp.w[t]});
    acc = acc < 0 ? term : c.ew(SOUFFLE_EW_ADD, {acc, term});
  }
  if (!c.ok) return no("not an MBConv program (depthwise)");
  int64_t stride = 1;
  if (c.peek() && c.peek()->op == SOUFFLE_OP_SLICE) {
    const Node* sl = c.take(SOUFFLE_OP_SLICE);
    if (sl->in[0] != acc || sl->begin != std::vector<int64_t>{0, 0, 0} || sl->end != std::vector<int64_t>{H, H, E} ||
        sl->stride != std::vector<int64_t>{2, 2, 1} || H % 2)
      return no("depthwise stride");
    acc = c.id();
    stride = 2;
  }
  const int64_t Ho = H / stride;
  int d = c.bn(c.reshape(acc, {Ho * Ho, E}), E, &mp.sd, &mp.bd, true);
  // squeeze-and-excitation
  const Node* rd = c.take(SOUFFLE_OP_REDUCE);
  if (!rd || rd->fn != SOUFFLE_RED_MEAN || rd->in[0] != d || rd->axis != 0 || !rd->keepdim)
    return no("not an MBConv program (pool)");
  const int pool = c.id();
  if (!c.peek() || c.peek()->op != SOUFFLE_OP_PLACEHOLDER || c.peek()->shape.size() != 2) return no("SE fc1");
  const int64_t S = c.peek()->shape[0];
  mp.W1 = c.ph({S, E});
  int h = c.mm(pool, mp.W1);
  mp.b1 = c.ph({S});
  h = c.ew(SOUFFLE_EW_ADD, {h, mp.b1});
  h = c.ew(SOUFFLE_EW_MUL, {h, c.ew(SOUFFLE_EW_SIGMOID, {h})});
  mp.W2 = c.ph({E, S});
  int gt = c.mm(h, mp.W2);
  mp.b2 = c.ph({E});
  gt = c.ew(SOUFFLE_EW_SIGMOID, {c.ew(SOUFFLE_EW_ADD, {gt, mp.b2})});
  d = c.ew(SOUFFLE_EW_MUL, {d, gt});
  // 1x1 project convolution (+ residual)
  if (!c.peek() || c.peek()->op != SOUFFLE_OP_PLACEHOLDER || c.peek()->shape.size() != 2) return no("project");
  const int64_t cout = c.peek()->shape[0];
  mp.Wp = c.ph({cout, E});
  int y = c.bn(c.mm(d, mp.Wp), cout, &mp.sp, &mp.bp, false);
  if (c.ok && c.peek()) {
    y = c.ew(SOUFFLE_EW_ADD, {y, mp.x});
    mp.residual = 1;
    if (stride != 1 || cout != cin) return no("residual shape");
  }
  if (!c.ok || c.i != N.size()) return no("not an MBConv program");
  if (g.outputs.size() != 1 || g.outputs[0] != y) return no("the only output must be the block output");
  if (E > MB_MAX_E) return no("too many expanded channels");
  const int sms = dev.num_sms > 0 ? dev.num_sms : 148;
  mp.y = y;
  mp.H = (int)H; mp.cin = (int)cin; mp.E = (int)E; mp.k = (int)k; mp.stride = (int)stride; mp.S = (int)S;
  mp.cout = (int)cout; mp.grid = sms; mp.num_sp = an.num_sp;
  // data reuse (Fig. 5(d)): the CTA's d block and the whole Wp in shared memory, when Wp is small and
  // each CTA owns enough pixels for the saved d round trip to outweigh staging Wp (measured: it pays
  // at 85 pixels per CTA, is neutral at 22 and costs at 6, profiles/r02_mbconv_ablation.jsonl)
  mp.pix_blk = (int)((Ho * Ho + sms - 1) / sms);
  mp.reuse = flags == 0 && mp.pix_blk >= 16 && (size_t)cout * E * 4 <= 64 * 1024 &&
             mbconv_reuse_smem(mp.pix_blk, (int)E, (int)cout) <= (size_t)MB_MAX_REUSE_SMEM;
  int64_t o = 0;
  mp.o_ctrl = o; o = al(o + 256, 256);
  mp.o_a = o; o = al(o + 4 * (mp.We >= 0 ? HW * E : 0), 256);
  mp.o_d = o; o = al(o + 4 * Ho * Ho * E, 256);
  mp.o_part = o; o = al(o + 4LL * sms * E, 256);
  mp.o_pooled = o; o = al(o + 4 * E, 256);
  mp.o_h = o; o = al(o + 4 * S, 256);
  mp.o_acc = o; o = al(o + 4 * Ho * Ho * cout, 256);
  mp.total = al(o, 4096);
  mp.on = true;
}

std::string mbconv_describe(const MbPlan& mp) {
  std::ostringstream os;
  if (!mp.on) {
    os << "pattern mbconv: not used (" << mp.why_not << ")\n";
    return os.str();
  }
  os << "pattern mbconv: " << mp.cin << " -> " << mp.cout << " channels, expand " << mp.E / mp.cin << ", depthwise "
     << mp.k << "x" << mp.k << " stride " << mp.stride << ", " << mp.H << "x" << mp.H << ", SE " << mp.S
     << (mp.residual ? ", residual" : "") << " -> 1 persistent launch (kernels/mbconv.cu), "
     << (mp.reuse ? "d reused from shared memory (Fig. 5(d)), " : "d through L2 (Fig. 5(c)), ") << mp.grid
     << " CTAs, 4-5 grid barriers (the partition's " << mp.num_sp << " subprogram(s) end at barriers of the launch)\n";
  return os.str();
}

souffle_status mbconv_run(Plan& p, void* ws, void* stream) {
  const MbPlan& mp = p.mb;
  auto ptr = [&](int node) -> const float* { return node < 0 ? nullptr : (const float*)p.buf_ptr[p.node_buf[node]]; };
  char* base = (char*)ws;
  MbParams prm{};
  prm.x = ptr(mp.x); prm.We = ptr(mp.We); prm.se = ptr(mp.se); prm.be = ptr(mp.be);
  for (int t = 0; t < MB_MAX_TAPS; ++t) {
    prm.w[t] = ptr(mp.w[t]);
    prm.m[t] = ptr(mp.m[t]);
  }
  prm.sd = ptr(mp.sd); prm.bd = ptr(mp.bd); prm.W1 = ptr(mp.W1); prm.b1 = ptr(mp.b1); prm.W2 = ptr(mp.W2);
  prm.b2 = ptr(mp.b2); prm.Wp = ptr(mp.Wp); prm.sp = ptr(mp.sp); prm.bp = ptr(mp.bp);
  prm.y = (float*)p.buf_ptr[p.node_buf[mp.y]];
  prm.a = (float*)(base + mp.o_a);
  prm.d = (float*)(base + mp.o_d);
  prm.pooled = (float*)(base + mp.o_pooled);
  prm.h = (float*)(base + mp.o_h);
  prm.acc = (float*)(base + mp.o_acc);
  prm.ctrl = (unsigned*)(base + mp.o_ctrl);
  if (std::getenv("SOUFFLE_MB_PROF")) prm.prof = (unsigned long long*)(base + mp.o_ctrl + 64);   // 8 stamps
  prm.H = mp.H; prm.cin = mp.cin; prm.E = mp.E; prm.k = mp.k; prm.stride = mp.stride; prm.S = mp.S;
  prm.cout = mp.cout; prm.residual = mp.residual; prm.reuse = mp.reuse; prm.pix_blk = mp.pix_blk;
  cudaError_t e = mbconv_launch(prm, mp.grid, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("mbconv launch: ") + cudaGetErrorString(e));
  return SOUFFLE_OK;
}

}  // namespace souffle
