// Swin Transformer pattern: strict TE-pattern match, workspace layout, the quasi-affine index maps
// (cyclic shift + window partition / reverse, patch merging) as int32 row maps, the launch sequence
// of the fused-subprogram kernels (kernels/swin.cu) and its CUDA-graph capture.
//
// Per block (Table 2; models.swin):
//   ROW   LN1 of the token rows gathered in window order through roll(-s) + window partition (§6.2)
//   GEMM  QKV + bias, q * d^-1/2, scatter to per-(window, head) Q / K / V^T tiles (reshape, permute
//         and slice TEs folded into the store: the vertical transformation)
//   ATTN  QK^T + relative-position bias (+ shift mask) -> softmax -> PV (Fig. 1(c) fused reductions)
//   GEMM  proj + bias + residual through window reverse + roll(+s) (the inverse map, same rows)
//   ROW   LN2;  GEMM FC1 + bias + GELU;  GEMM FC2 + bias + residual
// patch merging: ROW (2x2 gather + LN over 4C) + GEMM;  patch embedding: im2col + GEMM (+bias) +
// ROW (LN);  classifier: HEAD (LN + mean pool + linear).
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <sstream>
#include <string>

#include <cuda.h>
#include <cuda_runtime.h>

#include "plan.h"
#include "swin.h"

namespace souffle {

extern thread_local std::string g_err;
souffle_status fail(souffle_status c, const std::string& m);
cudaError_t sw_launch_gemm(const void* ta, const void* tb, const SwGemm& g, int grid, cudaStream_t s);
cudaError_t sw_launch_gemm2(const void* ta, const void* tb, const SwGemm& g, int grid, cudaStream_t s);
cudaError_t sw_launch_attn(const void* tq, const void* tk, const void* tv, const SwAttn& at, int grid, cudaStream_t s);
cudaError_t sw_launch_row(const SwRow& r, cudaStream_t s);
cudaError_t sw_launch_im2col(const SwIm2col& p, cudaStream_t s);
cudaError_t sw_launch_head(const SwHead& h, cudaStream_t s);
cudaError_t sw_launch_bias(const SwBias& b, int max_table, cudaStream_t s);
cudaError_t sw_launch_pool(const SwHead& h, cudaStream_t s);

namespace {

// strict cursor over the node list in builder order
struct Cur {
  const Graph& g;
  size_t i = 0;
  bool ok = true;
  explicit Cur(const Graph& gr) : g(gr) {}
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
  int red(int fn, int in, int axis, int keepdim) {
    const Node* n = next(SOUFFLE_OP_REDUCE);
    if (!n || n->fn != fn || n->in[0] != in || n->axis != axis || n->keepdim != keepdim) { ok = false; return -1; }
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
  int roll(int in, std::vector<int64_t> shifts) {
    const Node* n = next(SOUFFLE_OP_ROLL);
    if (!n || n->in[0] != in || n->shifts != shifts) { ok = false; return -1; }
    return id();
  }
  int slice(int in, std::vector<int64_t> b, std::vector<int64_t> e, std::vector<int64_t> s) {
    const Node* n = next(SOUFFLE_OP_SLICE);
    if (!n || n->in[0] != in || n->begin != b || n->end != e || n->stride != s) { ok = false; return -1; }
    return id();
  }
};

int match_ln(Cur& c, int x, int64_t H, int* gm, int* be, double* eps) {
  int mu = c.red(SOUFFLE_RED_MEAN, x, 1, 1);
  int d = c.ew(SOUFFLE_EW_SUB, {x, mu});
  int q = c.ew(SOUFFLE_EW_MUL, {d, d});
  int v = c.red(SOUFFLE_RED_MEAN, q, 1, 1);
  int ve = c.ews(SOUFFLE_EW_ADD_SCALAR, v, eps);
  int rs = c.ew(SOUFFLE_EW_RSQRT, {ve});
  int n = c.ew(SOUFFLE_EW_MUL, {d, rs});
  *gm = c.ph({H}, SOUFFLE_F32);
  int a = c.ew(SOUFFLE_EW_MUL, {n, *gm});
  *be = c.ph({H}, SOUFFLE_F32);
  return c.ew(SOUFFLE_EW_ADD, {a, *be});
}

int64_t al(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

// window-order GEMM row -> token row of the (rolled) feature map: roll(-s) then window partition
void window_map(int B, int R, int w, int s, std::vector<int32_t>& out) {
  const int n = R / w, L2 = w * w;
  for (int64_t r = 0; r < (int64_t)B * R * R; ++r) {
    const int64_t win = r / L2;
    const int i = (int)(r % L2);
    const int b = (int)(win / (n * n)), wy = (int)(win / n % n), wx = (int)(win % n);
    const int y = wy * w + i / w, x = wx * w + i % w;
    out.push_back((int32_t)((int64_t)b * R * R + ((y + s) % R) * R + (x + s) % R));
  }
}
// patch merging: output row (b, yy, xx), channel segment s = kx * 2 + ky (torchvision x0..x3 order)
void merge_map(int B, int R, std::vector<int32_t>& out) {
  const int h = R / 2;
  for (int b = 0; b < B; ++b)
    for (int yy = 0; yy < h; ++yy)
      for (int xx = 0; xx < h; ++xx)
        for (int s = 0; s < 4; ++s) {
          const int kx = s >> 1, ky = s & 1;
          out.push_back((int32_t)((int64_t)b * R * R + (2 * yy + ky) * R + (2 * xx + kx)));
        }
}

}  // namespace

void swin_match(const Graph& g, const souffle_device_desc& dev, uint32_t flags, SwinPlan& sp) {
  sp = SwinPlan();
  auto no = [&](const char* why) { sp.on = false; sp.why_not = why; };
  if (flags != 0) return no("ablation flags select the generic executor");
  const auto& N = g.nodes;
  if (N.size() < 40 || N[0].op != SOUFFLE_OP_PLACEHOLDER || N[0].is_const || N[0].shape.size() != 4 ||
      N[0].dtype != SOUFFLE_F32 || N[0].shape[1] != 3 || N[0].shape[2] != N[0].shape[3])
    return no("first node is not an fp32 [B, 3, H, H] image");
  const int64_t B = N[0].shape[0], img = N[0].shape[2];
  Cur c(g);
  c.i = 1;
  // ---- patch embedding: reshape (B,3,R,p,R,p) -> permute -> reshape -> GEMM + bias -> LN
  const Node& r0 = N[1];
  if (r0.op != SOUFFLE_OP_RESHAPE || r0.shape.size() != 6) return no("no patch-embedding reshape");
  const int64_t R = r0.shape[2], p = r0.shape[3];
  if (R * p != img) return no("patch grid");
  int t = c.reshape(0, {B, 3, R, p, R, p});
  t = c.reshape(c.permute(t, {0, 2, 4, 1, 3, 5}), {B * R * R, 3 * p * p});
  if (!c.ok || c.i >= N.size() || N[c.i].op != SOUFFLE_OP_PLACEHOLDER || N[c.i].shape.size() != 2) return no("Wpe");
  const int64_t C0 = N[c.i].shape[0];
  sp.Wpe = c.ph({C0, 3 * p * p}, SOUFFLE_BF16);
  int pe = c.mm(t, sp.Wpe, 1);
  sp.bpe = c.ph({C0}, SOUFFLE_F32);
  pe = c.ew(SOUFFLE_EW_ADD, {pe, sp.bpe});
  double eps = 0;
  int h = match_ln(c, pe, C0, &sp.gpe, &sp.bepe, &eps);
  if (!c.ok) return no("patch embedding");
  // ---- stages of blocks, separated by patch merging
  int64_t C = C0, Rs = R, w = 0;
  int stage = 0;
  while (c.ok && c.i < N.size()) {
    const Node& nx = N[c.i];
    // the final LayerNorm: its 11 TEs are followed by reshape (B, R*R, C) and a keepdim-0 mean
    if (nx.op == SOUFFLE_OP_REDUCE && c.i + 12 < N.size() && N[c.i + 11].op == SOUFFLE_OP_RESHAPE &&
        N[c.i + 11].shape.size() == 3 && N[c.i + 12].op == SOUFFLE_OP_REDUCE && !N[c.i + 12].keepdim)
      break;
    if (nx.op == SOUFFLE_OP_RESHAPE && nx.shape.size() == 6 && nx.shape[2] == 2) {
      // patch merging
      SwinMergeIds mg;
      int m = c.reshape(h, {B, Rs / 2, 2, Rs / 2, 2, C});
      m = c.reshape(c.permute(m, {0, 1, 3, 4, 2, 5}), {B * (Rs / 2) * (Rs / 2), 4 * C});
      double e2 = 0;
      m = match_ln(c, m, 4 * C, &mg.g, &mg.be, &e2);
      mg.W = c.ph({2 * C, 4 * C}, SOUFFLE_BF16);
      h = c.mm(m, mg.W, 1);
      if (!c.ok || e2 != eps || Rs % 2) return no("patch merging");
      sp.merges.push_back(mg);
      C *= 2;
      Rs /= 2;
      ++stage;
      continue;
    }
    // ---- one block
    SwinBlockIds bk;
    bk.stage = stage;
    double e1 = 0, e2 = 0;
    const int x = h;
    int l1 = match_ln(c, x, C, &bk.g1, &bk.be1, &e1);
    int tt = c.reshape(l1, {B, Rs, Rs, C});
    if (c.ok && c.i < N.size() && N[c.i].op == SOUFFLE_OP_ROLL) {
      const Node& rl = N[c.i];
      // roll TEs store shifts normalised to [0, n): roll(-s) on an R x R map is R - s
      if (rl.shifts.size() != 4 || rl.shifts[1] == 0 || rl.shifts[1] != rl.shifts[2]) return no("roll");
      bk.shift = (int)(Rs - rl.shifts[1]);
      tt = c.roll(tt, {0, Rs - bk.shift, Rs - bk.shift, 0});
    }
    if (!c.ok || c.i >= N.size() || N[c.i].op != SOUFFLE_OP_RESHAPE || N[c.i].shape.size() != 6) return no("window partition");
    w = N[c.i].shape[2];
    const int64_t n = Rs / w, nW = n * n, L2 = w * w;
    if (bk.shift && bk.shift != w / 2) return no("shift must be window / 2 (torchvision)");
    tt = c.reshape(tt, {B, n, w, n, w, C});
    tt = c.reshape(c.permute(tt, {0, 1, 3, 2, 4, 5}), {B * nW * L2, C});
    bk.Wqkv = c.ph({3 * C, C}, SOUFFLE_BF16);
    int qkv = c.mm(tt, bk.Wqkv, 1);
    bk.bqkv = c.ph({3 * C}, SOUFFLE_F32);
    qkv = c.ew(SOUFFLE_EW_ADD, {qkv, bk.bqkv});
    if (!c.ok || c.i >= N.size() || N[c.i].op != SOUFFLE_OP_RESHAPE || N[c.i].shape.size() != 5) return no("qkv reshape");
    const int64_t nh = N[c.i].shape[3], d = C / nh;
    qkv = c.permute(c.reshape(qkv, {B * nW, L2, 3, nh, d}), {2, 0, 3, 1, 4});
    int qkvs[3];
    for (int j = 0; j < 3; ++j)
      qkvs[j] = c.reshape(c.slice(qkv, {j, 0, 0, 0, 0}, {j + 1, B * nW, nh, L2, d}, {1, 1, 1, 1, 1}), {B * nW, nh, L2, d});
    double qs = 0;
    int q = c.ews(SOUFFLE_EW_MUL_SCALAR, qkvs[0], &qs);
    if (c.ok && std::fabs(qs - std::pow((double)d, -0.5)) > 1e-12) return no("q scale is not d^-1/2");
    int a = c.mm(q, qkvs[1], 1);
    bk.bias = c.ph({nh, L2, L2}, SOUFFLE_F32);
    a = c.ew(SOUFFLE_EW_ADD, {a, bk.bias});
    if (bk.shift) {
      a = c.reshape(a, {B, nW, nh, L2, L2});
      bk.mask = c.ph({nW, 1, L2, L2}, SOUFFLE_F32);
      a = c.reshape(c.ew(SOUFFLE_EW_ADD, {a, bk.mask}), {B * nW, nh, L2, L2});
    }
    int mx = c.red(SOUFFLE_RED_MAX, a, 3, 1);
    int e = c.ew(SOUFFLE_EW_EXP, {c.ew(SOUFFLE_EW_SUB, {a, mx})});
    int z = c.red(SOUFFLE_RED_SUM, e, 3, 1);
    int pr = c.ew(SOUFFLE_EW_DIV, {e, z});
    int o = c.mm(pr, qkvs[2], 0);
    o = c.reshape(c.permute(o, {0, 2, 1, 3}), {B * nW * L2, C});
    bk.Wp = c.ph({C, C}, SOUFFLE_BF16);
    o = c.mm(o, bk.Wp, 1);
    bk.bp = c.ph({C}, SOUFFLE_F32);
    o = c.ew(SOUFFLE_EW_ADD, {o, bk.bp});
    o = c.reshape(c.permute(c.reshape(o, {B, n, n, w, w, C}), {0, 1, 3, 2, 4, 5}), {B, Rs, Rs, C});
    if (bk.shift) o = c.roll(o, {0, bk.shift, bk.shift, 0});
    int x1 = c.ew(SOUFFLE_EW_ADD, {x, c.reshape(o, {B * Rs * Rs, C})});
    int l2 = match_ln(c, x1, C, &bk.g2, &bk.be2, &e2);
    if (!c.ok || c.i >= N.size() || N[c.i].op != SOUFFLE_OP_PLACEHOLDER || N[c.i].shape.size() != 2) return no("W1");
    const int64_t F = N[c.i].shape[0];
    bk.W1 = c.ph({F, C}, SOUFFLE_BF16);
    int f = c.mm(l2, bk.W1, 1);
    bk.b1 = c.ph({F}, SOUFFLE_F32);
    f = c.ew(SOUFFLE_EW_GELU_ERF, {c.ew(SOUFFLE_EW_ADD, {f, bk.b1})});
    bk.W2 = c.ph({C, F}, SOUFFLE_BF16);
    f = c.mm(f, bk.W2, 1);
    bk.b2 = c.ph({C}, SOUFFLE_F32);
    f = c.ew(SOUFFLE_EW_ADD, {f, bk.b2});
    h = c.ew(SOUFFLE_EW_ADD, {x1, f});
    if (!c.ok) return no("TE program is not a Swin block sequence");
    if (e1 != eps || e2 != eps) return no("LayerNorm eps differs");
    if (d != 32 || w != 7 || C % 128 || Rs % w || nh % 2 || F != sp.mlp * C)
      return no("needs head dim 32, window 7, C % 128 == 0, MLP ratio 4");
    if ((int)sp.depths.size() <= stage) {
      sp.depths.push_back(0);
      sp.heads.push_back((int)nh);
    }
    if (sp.heads[stage] != nh) return no("heads differ inside a stage");
    sp.depths[stage]++;
    sp.blocks.push_back(bk);
  }
  // ---- final LN + mean pool + classifier
  double ef = 0;
  int hf = match_ln(c, h, C, &sp.gn, &sp.ben, &ef);
  hf = c.red(SOUFFLE_RED_MEAN, c.reshape(hf, {B, Rs * Rs, C}), 1, 0);
  if (!c.ok || c.i >= N.size() || N[c.i].op != SOUFFLE_OP_PLACEHOLDER) return no("classifier");
  const int64_t classes = N[c.i].shape[0];
  sp.Wh = c.ph({classes, C}, SOUFFLE_BF16);
  int y = c.mm(hf, sp.Wh, 1);
  sp.bh = c.ph({classes}, SOUFFLE_F32);
  y = c.ew(SOUFFLE_EW_ADD, {y, sp.bh});
  if (!c.ok || c.i != N.size() || ef != eps) return no("TE program is not a Swin Transformer");
  if (g.outputs.size() != 1 || g.outputs[0] != y) return no("the only output must be the logits");
  if (sp.blocks.empty() || (int)sp.merges.size() + 1 != (int)sp.depths.size()) return no("stage structure");
  if (p != 4 || C0 % 128 || C > 1024 || 4 * (C / 2) > 2048) return no("patch size 4 / widths");
  sp.B = (int)B; sp.img = (int)img; sp.patch = (int)p; sp.C0 = (int)C0; sp.window = (int)w;
  sp.classes = (int)classes; sp.eps = eps; sp.X = 0; sp.Y = y;
  sp.num_sms = dev.num_sms > 0 ? dev.num_sms : 148;
  // ---- workspace layout
  const int64_t T1 = B * R * R;
  int64_t qk = 0;
  {
    int64_t Ts = T1;
    for (size_t s = 0; s < sp.depths.size(); ++s, Ts /= 4) qk = std::max(qk, Ts / (w * w) * sp.heads[s] * 64 * 32);
  }
  int64_t o = 0;
  auto take = [&](int64_t bytes) { int64_t r = o; o = al(o + bytes, 1024); return r; };
  sp.o_x0 = take(T1 * C0 * 4);
  sp.o_x1 = take(T1 * C0 * 4);
  sp.o_a = take(T1 * std::max<int64_t>(C0, 64) * 2);
  sp.o_ctx = take(T1 * C0 * 2);
  sp.o_h = take(T1 * 4 * C0 * 2);
  sp.o_q = take(qk * 2);
  sp.o_k = take(qk * 2);
  sp.o_vt = take(qk * 2);
  sp.o_wpad = take(C0 * 64 * 2);
  sp.o_pool = take(B * 1024 * 4);
  sp.o_trace = take(8 * 1024);
  // split-K partials / counters (a split GEMM has at most num_sms units of 128 x 256 fp32)
  sp.o_part = take((int64_t)sp.num_sms * 128 * 256 * 4);
  sp.o_cnt = take((int64_t)2 * sp.num_sms * 4 + 256);
  // per-block score-bias tables [nW or 1][heads][SW_TAB] (rebuilt from the bound bias / mask by the
  // first launch of every run) and their descriptor list
  {
    int64_t tabs = 0, Rr = R;
    size_t gb = 0;
    for (size_t s2 = 0; s2 < sp.depths.size(); ++s2, Rr /= 2)
      for (int j = 0; j < sp.depths[s2]; ++j, ++gb) {
        const int64_t nWe = sp.blocks[gb].mask >= 0 ? (Rr / w) * (Rr / w) : 1;
        tabs += nWe * sp.heads[s2] * SW_TAB;
      }
    sp.o_tab = take(tabs * 4);
    sp.tab_floats = tabs;
    sp.o_tabent = take((int64_t)sp.blocks.size() * (int64_t)sizeof(SwBiasEnt));
  }
  // index maps: per stage the unshifted and shifted window maps, then the merge maps
  sp.maps.clear();
  {
    int64_t Rr = R;
    for (size_t s = 0; s < sp.depths.size(); ++s, Rr /= 2) {
      window_map((int)B, (int)Rr, (int)w, 0, sp.maps);
      window_map((int)B, (int)Rr, (int)w, (int)(w / 2), sp.maps);
      if (s + 1 < sp.depths.size()) merge_map((int)B, (int)Rr, sp.maps);
    }
  }
  sp.o_maps = take((int64_t)sp.maps.size() * 4);
  sp.total = al(o, 4096);
  sp.on = true;
}

std::string swin_describe(const SwinPlan& sp) {
  std::ostringstream os;
  if (!sp.on) {
    os << "pattern swin: not used (" << sp.why_not << ")\n";
    return os.str();
  }
  os << "pattern swin: batch " << sp.B << ", " << sp.img << "x" << sp.img << ", embed " << sp.C0 << ", depths";
  for (int d : sp.depths) os << " " << d;
  os << ", heads";
  for (int h : sp.heads) os << " " << h;
  os << " -> " << sp.launches << " launches of kernels/swin.cu (one CUDA graph): per block LN1-gather | "
        "QKV-gemm(+bias, q-scale, window scatter) | window-attention(tcgen05, bias+mask) | proj-gemm(+bias, "
        "window-reverse residual) | LN2 | FC1-gemm(+bias, GELU) | FC2-gemm(+bias, residual)\n";
  return os.str();
}

// ------------------------------------------------------------------ runtime
namespace {
typedef CUresult (*EncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiled encoder() {
  static EncodeTiled fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult qr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &qr) == cudaSuccess &&
        qr == cudaDriverEntryPointSuccess)
      fn = (EncodeTiled)p;
  }
  return fn;
}
// bf16 [rows][cols] row-major, box {box_cols, box_rows}
bool make_map(CUtensorMap* m, void* ptr, int64_t rows, int64_t cols, int box_rows, int box_cols, int swz) {
  EncodeTiled enc = encoder();
  if (!enc) return false;
  cuuint64_t d[2] = {(cuuint64_t)cols, (cuuint64_t)rows}, st[1] = {(cuuint64_t)cols * 2};
  cuuint32_t bx[2] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows}, es[2] = {1, 1};
  CUtensorMapSwizzle sw = swz == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : swz == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                                              : CU_TENSOR_MAP_SWIZZLE_NONE;
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, ptr, d, st, bx, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
struct Launcher {
  CUtensorMap maps[3];
};
}  // namespace

int sw_gemm_smem(int BN, int stages);
int sw_attn_smem();

// the launch sequence with resolved pointers; `maps` receives the encoded tensor maps of each op
static souffle_status build_ops(Plan& p, char* base, std::vector<SwinOp>& ops, std::vector<Launcher>& tm) {
  SwinPlan& sp = p.swin;
  auto bound = [&](int node) -> char* { return (char*)p.buf_ptr[p.node_buf[node]]; };
  auto fptr = [&](int node) { return (const float*)bound(node); };
  const int B = sp.B, w = sp.window, L2 = w * w, nsm = sp.num_sms;
  const int64_t R1 = sp.img / sp.patch;
  float* x[2] = {(float*)(base + sp.o_x0), (float*)(base + sp.o_x1)};
  uint16_t* abuf = (uint16_t*)(base + sp.o_a);
  uint16_t* ctx = (uint16_t*)(base + sp.o_ctx);
  uint16_t* hbuf = (uint16_t*)(base + sp.o_h);
  uint16_t* qb = (uint16_t*)(base + sp.o_q);
  uint16_t* kb = (uint16_t*)(base + sp.o_k);
  uint16_t* vtb = (uint16_t*)(base + sp.o_vt);
  uint16_t* wpad = (uint16_t*)(base + sp.o_wpad);
  const int32_t* maps = (const int32_t*)(base + sp.o_maps);
  ops.clear();
  tm.clear();
  float* tabs = (float*)(base + sp.o_tab);
  SwBiasEnt* tabent = (SwBiasEnt*)(base + sp.o_tabent);
  std::vector<float*> block_tab;
  std::vector<int> block_nw;
  {
    SwinOp op;
    op.kind = SW_BIAS;
    int64_t off = 0, Rr = R1;
    size_t gb2 = 0;
    sp.tabent.clear();
    for (size_t s2 = 0; s2 < sp.depths.size(); ++s2, Rr /= 2)
      for (int j = 0; j < sp.depths[s2]; ++j, ++gb2) {
        const SwinBlockIds& bk = sp.blocks[gb2];
        SwBiasEnt e{};
        e.bias = fptr(bk.bias);
        e.mask = bk.mask >= 0 ? fptr(bk.mask) : nullptr;
        e.dst = tabs + off;
        e.heads = sp.heads[s2];
        e.nW = bk.mask >= 0 ? (int)((Rr / w) * (Rr / w)) : 1;
        e.first = (int32_t)off;
        sp.tabent.push_back(e);
        block_tab.push_back(tabs + off);
        block_nw.push_back(e.nW);
        off += (int64_t)e.nW * e.heads * SW_TAB;
      }
    int64_t mx = 0;
    for (auto& e : sp.tabent) mx = std::max<int64_t>(mx, (int64_t)e.nW * e.heads * SW_TAB);
    op.grid = (int)std::min<int64_t>(mx, 1 << 30);   // largest table (elements): sizes the launch
    op.bias.ent = tabent;
    op.bias.n = (int)sp.tabent.size();
    op.bias.total = (int32_t)off;
    op.bias.L2 = L2;
    ops.push_back(op);
    tm.push_back(Launcher{});
  }
  auto gemm = [&](void* A, int64_t M, int64_t K, void* W, int64_t N, int epi) -> SwinOp& {
    SwinOp op;
    op.kind = SW_GEMM;
    SwGemm& g = op.gemm;
    std::memset(&g, 0, sizeof(g));
    g.M = (int)M; g.N = (int)N; g.K = (int)K; g.epi = epi;
    if (const char* e = std::getenv("SOUFFLE_SWIN_EPI_DIRECT")) g.direct = std::atoi(e) != 0;   // A/B studies
    // tile policy: the widest N tile (smem operand bandwidth per MMA) that still fills the SMs;
    // with too few output tiles (small M, e.g. batch 1) the K loop is split across CTAs
    const int64_t mt = (M + 127) / 128, nk = K / 64;
    g.BN = 64;
    for (int bn : {256, 128}) {
      if (N % bn == 0 && mt * (N / bn) >= nsm) { g.BN = bn; break; }
    }
    if (g.BN == 64 && N % 64) g.BN = N % 128 == 0 ? 128 : 256;
    // narrow outputs (proj, fc2, patch merge: 256 <= N <= 1024) take 128-wide tiles: with 256 their tile count
    // lands just above one wave (b64: 196 tiles on 148 SMs), with 64 the residual epilogue's row
    // traffic per MMA doubles -- measured at b8 / b64 (profiles/r02_swin_bn_study.txt); small M keeps
    // the split-K policy (batch 1 measured slower with 128)
    if (N >= 256 && N <= 1024 && N % 128 == 0 && mt >= 8 && g.BN != 128 && !std::getenv("SOUFFLE_SWIN_BN_OLD")) g.BN = 128;
    if (const char* e = std::getenv("SOUFFLE_SWIN_BN")) {   // tile studies: force the N tile where it divides N
      const int bn = std::atoi(e);
      if ((bn == 64 || bn == 128 || bn == 256) && N % bn == 0) g.BN = bn;
    }
    g.stages = g.BN == 256 ? 4 : g.BN == 128 ? 6 : 8;
    const int tiles = (int)(N / g.BN * mt);
    g.splits = 1;
    // split K only when a CTA would otherwise stream more than ~256 KB of operands: the split's
    // partial round trip through L2 costs a few microseconds of latency.  Residual epilogues add
    // their partials with atomics (no round trip), so they split down to ~96 KB per CTA
    const int64_t cap = epi == SWE_RESID ? 96 * 1024 : 256 * 1024;
    for (int sp2 = 1; sp2 <= 16 && nk % sp2 == 0 && tiles * sp2 <= nsm; sp2 *= 2) {
      g.splits = sp2;
      if ((128 + g.BN) * 2 * K / sp2 <= cap) break;
    }
    g.part = (float*)(base + sp.o_part);
    g.cnt = (unsigned*)(base + sp.o_cnt);
    op.grid = g.splits > 1 ? tiles * g.splits : std::min(tiles, nsm);
    // large M: 256 x 256 tiles on CTA pairs (tcgen05 cta_group::2) when there are enough of them to
    // fill every pair of SMs.  Opt-in (SOUFFLE_SWIN_2SM=1): parity-green (b8 / b64 tests), but on this
    // pool it measured within +-4 % of the 1-SM tiles at batch 64 -- these GEMMs are bound by the L2
    // bandwidth of re-streamed operands and the GELU epilogue, not by per-SM operand ingest
    const int64_t t2 = (M + 255) / 256 * (N / 256);
    const char* e2 = std::getenv("SOUFFLE_SWIN_2SM");
    op.two_sm = N % 256 == 0 && t2 >= nsm / 2 && e2 && std::atoi(e2) != 0;
    int wbox = g.BN;
    if (op.two_sm) {
      g.BN = 256;
      g.splits = 1;
      g.stages = 6;
      op.grid = 2 * (int)std::min<int64_t>(t2, nsm / 2);
      wbox = 128;   // each CTA of the pair loads half of the 256 W rows
    }
    Launcher L;
    if (!make_map(&L.maps[0], A, M, K, 128, 64, 128) || !make_map(&L.maps[1], W, N, K, wbox, 64, 128)) op.grid = -1;
    ops.push_back(op);
    tm.push_back(L);
    return ops.back();
  };
  auto row = [&](const float* xin, const int32_t* src, int nsrc, int64_t rows, int64_t cols, int gm, int be,
                 uint16_t* ob, float* of) {
    SwinOp op;
    op.kind = SW_ROW;
    SwRow& r = op.row;
    r.rows = (int)rows; r.cols = (int)cols; r.nsrc = nsrc; r.x = xin; r.src = src;
    r.gamma = fptr(gm); r.beta = fptr(be); r.eps = (float)sp.eps; r.out_b = ob; r.out_f = of;
    ops.push_back(op);
    tm.push_back(Launcher{});
  };
  // ---- patch embedding: im2col -> GEMM + bias (fp32, x[1]) -> LN -> x[0]
  {
    SwinOp op;
    op.kind = SW_IM2COL;
    SwIm2col& m = op.im2col;
    m.B = B; m.img = sp.img; m.p = sp.patch; m.R = (int)R1; m.C = sp.C0;
    m.image = fptr(sp.X); m.out = abuf; m.w = (const uint16_t*)bound(sp.Wpe); m.wpad = wpad;
    ops.push_back(op);
    tm.push_back(Launcher{});
    const int64_t T1 = (int64_t)B * R1 * R1;
    SwinOp& g = gemm(abuf, T1, 64, wpad, sp.C0, SWE_F32);
    g.gemm.bias = fptr(sp.bpe);
    g.gemm.out_f = x[1];
    row(x[1], nullptr, 1, T1, sp.C0, sp.gpe, sp.bepe, nullptr, x[0]);
  }
  int cur = 0, gb = 0;
  int64_t R = R1, C = sp.C0, moff = 0;
  for (size_t s = 0; s < sp.depths.size(); ++s) {
    const int64_t T = (int64_t)B * R * R, n = R / w, nW = n * n, nh = sp.heads[s], units = T / L2 * nh;
    const int32_t* wmap[2] = {maps + moff, maps + moff + T};
    const int32_t* mmap = maps + moff + 2 * T;
    for (int j = 0; j < sp.depths[s]; ++j, ++gb) {
      const SwinBlockIds& bk = sp.blocks[gb];
      const int32_t* map = wmap[bk.shift ? 1 : 0];
      row(x[cur], map, 1, T, C, bk.g1, bk.be1, abuf, nullptr);
      SwinOp& q = gemm(abuf, T, C, bound(bk.Wqkv), 3 * C, SWE_QKV);
      q.gemm.bias = fptr(bk.bqkv);
      q.gemm.q = qb; q.gemm.k = kb; q.gemm.vt = vtb;
      q.gemm.C = (int)C; q.gemm.heads = (int)nh; q.gemm.L2 = L2; q.gemm.qscale = (float)std::pow(32.0, -0.5);
      {
        SwinOp op;
        op.kind = SW_ATTN;
        SwAttn& a = op.attn;
        a.units = (int)units; a.heads = (int)nh; a.nW = block_nw[gb]; a.L2 = L2;
        a.tab = block_tab[gb]; a.ctx = ctx; a.C = (int)C;
        op.grid = (int)std::min<int64_t>(units / 2, 2 * nsm);
        Launcher L;
        if (!make_map(&L.maps[0], qb, units * 64, 32, 128, 32, 64) || !make_map(&L.maps[1], kb, units * 64, 32, 128, 32, 64) ||
            !make_map(&L.maps[2], vtb, units * 32, 64, 64, 64, 128))
          op.grid = -1;
        ops.push_back(op);
        tm.push_back(L);
      }
      SwinOp& pj = gemm(ctx, T, C, bound(bk.Wp), C, SWE_RESID);
      pj.gemm.bias = fptr(bk.bp);
      pj.gemm.out_f = x[cur];
      pj.gemm.rowmap = map;
      row(x[cur], nullptr, 1, T, C, bk.g2, bk.be2, abuf, nullptr);
      SwinOp& f1 = gemm(abuf, T, C, bound(bk.W1), 4 * C, SWE_GELU);
      f1.gemm.bias = fptr(bk.b1);
      f1.gemm.out_b = hbuf;
      SwinOp& f2 = gemm(hbuf, T, 4 * C, bound(bk.W2), C, SWE_RESID);
      f2.gemm.bias = fptr(bk.b2);
      f2.gemm.out_f = x[cur];
    }
    if (s + 1 < sp.depths.size()) {
      const SwinMergeIds& mg = sp.merges[s];
      row(x[cur], mmap, 4, T / 4, 4 * C, mg.g, mg.be, abuf, nullptr);
      SwinOp& m = gemm(abuf, T / 4, 4 * C, bound(mg.W), 2 * C, SWE_F32);
      m.gemm.out_f = x[cur ^ 1];
      cur ^= 1;
      moff += 3 * T;
      C *= 2;
      R /= 2;
    }
  }
  for (int k : {SW_POOL, SW_HEAD}) {
    SwinOp op;
    op.kind = k;
    SwHead& hd = op.head;
    hd.B = B; hd.L = (int)(R * R); hd.C = (int)C; hd.classes = sp.classes; hd.x = x[cur];
    hd.gamma = fptr(sp.gn); hd.beta = fptr(sp.ben); hd.eps = (float)sp.eps;
    hd.W = (const uint16_t*)bound(sp.Wh); hd.bias = fptr(sp.bh); hd.out = (float*)bound(sp.Y);
    hd.pooled = (float*)(base + sp.o_pool);
    ops.push_back(op);
    tm.push_back(Launcher{});
  }
  // debug trace (SOUFFLE_SWIN_TRACE=1): every launch stamps %globaltimer into the workspace
  unsigned long long* tr = std::getenv("SOUFFLE_SWIN_TRACE") ? (unsigned long long*)(base + sp.o_trace) : nullptr;
  for (size_t i = 0; i < ops.size(); ++i) {
    SwinOp& op = ops[i];
    const int k = (int)i;
    op.gemm.trace = op.attn.trace = op.row.trace = op.im2col.trace = op.head.trace = op.bias.trace = tr;
    op.gemm.op = op.attn.op = op.row.op = op.im2col.op = op.head.op = op.bias.op = k;
  }
  for (auto& op : ops)
    if (op.grid < 0) return fail(SOUFFLE_E_CUDA, "cuTensorMapEncodeTiled failed (pointer alignment?)");
  return SOUFFLE_OK;
}

static cudaError_t launch_ops(const std::vector<SwinOp>& ops, const std::vector<Launcher>& tm, cudaStream_t s) {
  cudaError_t e = cudaSuccess;
  for (size_t i = 0; i < ops.size() && e == cudaSuccess; ++i) {
    const SwinOp& op = ops[i];
    switch (op.kind) {
      case SW_IM2COL: e = sw_launch_im2col(op.im2col, s); break;
      case SW_ROW: e = sw_launch_row(op.row, s); break;
      case SW_GEMM:
        e = op.two_sm ? sw_launch_gemm2(&tm[i].maps[0], &tm[i].maps[1], op.gemm, op.grid, s)
                      : sw_launch_gemm(&tm[i].maps[0], &tm[i].maps[1], op.gemm, op.grid, s);
        break;
      case SW_ATTN: e = sw_launch_attn(&tm[i].maps[0], &tm[i].maps[1], &tm[i].maps[2], op.attn, op.grid, s); break;
      case SW_BIAS: e = sw_launch_bias(op.bias, op.grid, s); break;
      case SW_POOL: e = sw_launch_pool(op.head, s); break;
      default: e = sw_launch_head(op.head, s); break;
    }
  }
  return e;
}

souffle_status swin_init(Plan& p, void* ws, void* stream) {
  SwinPlan& sp = p.swin;
  char* base = (char*)ws;
  cudaStream_t s = (cudaStream_t)stream;
  std::vector<SwinOp> ops;
  std::vector<Launcher> tm;
  souffle_status st = build_ops(p, base, ops, tm);
  if (st != SOUFFLE_OK) return st;
  cudaError_t e = cudaMemsetAsync(base, 0, (size_t)sp.total, s);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(base + sp.o_maps, sp.maps.data(), sp.maps.size() * 4, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(base + sp.o_tabent, sp.tabent.data(), sp.tabent.size() * sizeof(SwBiasEnt),
                        cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("swin workspace init: ") + cudaGetErrorString(e));
  // capture the launch sequence once (kernel parameters hold the tensor maps and pointers)
  if (sp.graph_exec) {
    cudaGraphExecDestroy((cudaGraphExec_t)sp.graph_exec);
    sp.graph_exec = nullptr;
  }
  cudaStream_t cs;
  e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
  cudaGraph_t graph = nullptr;
  if (e == cudaSuccess) e = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal);
  if (e == cudaSuccess) {
    cudaError_t le = launch_ops(ops, tm, cs);
    e = cudaStreamEndCapture(cs, &graph);
    if (le != cudaSuccess) e = le;
  }
  cudaGraphExec_t exec = nullptr;
  if (e == cudaSuccess) e = cudaGraphInstantiate(&exec, graph, 0);
  if (graph) cudaGraphDestroy(graph);
  cudaStreamDestroy(cs);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("swin graph capture: ") + cudaGetErrorString(e));
  sp.graph_exec = exec;
  sp.launches = (int)ops.size();
  p.inited_ws = ws;
  p.dirty = false;
  return SOUFFLE_OK;
}

souffle_status swin_run(Plan& p, void* ws, void* stream) {
  (void)ws;
  SwinPlan& sp = p.swin;
  if (!sp.graph_exec) return fail(SOUFFLE_E_STATE, "swin plan not initialised");
  cudaError_t e = cudaGraphLaunch((cudaGraphExec_t)sp.graph_exec, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("swin graph launch: ") + cudaGetErrorString(e));
  return SOUFFLE_OK;
}

int swin_launch_count(const SwinPlan& sp) {
  int n = 4 + 2;   // bias tables, im2col, embed GEMM, embed LN; pool, head
  for (size_t s = 0; s < sp.depths.size(); ++s) n += 7 * sp.depths[s] + (s + 1 < sp.depths.size() ? 2 : 0);
  return n;
}

}  // namespace souffle
