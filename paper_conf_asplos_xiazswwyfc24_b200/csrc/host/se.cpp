// EfficientNet squeeze-and-excitation pattern (Fig. 5 / 6): strict TE match, tile policy,
// workspace layout and launch of kernels/se.cu.
#include <algorithm>
#include <sstream>
#include <string>

#include <cuda_runtime.h>

#include "plan.h"
#include "se.h"

namespace souffle {

souffle_status fail(souffle_status c, const std::string& m);
cudaError_t se_launch(const SeParams& prm, int grid, cudaStream_t s);
size_t se_smem_bytes(const SeParams& p);

namespace {
int64_t al(int64_t x, int64_t a) { return (x + a - 1) / a * a; }
}  // namespace

void se_match(const Graph& g, const Analysis& an, const souffle_device_desc& dev, uint32_t flags, SePlan& sp) {
  sp = SePlan();
  auto no = [&](const char* why) { sp.on = false; sp.why_not = why; };
  if (flags != 0 && flags != SOUFFLE_FLAG_NO_PREFETCH) return no("ablation flags select the generic executor");
  const auto& N = g.nodes;
  // node order of models.se_module: x, mean, W1, mm, b1, add, sigmoid, mul, W2, mm, b2, add, sigmoid, mul
  if (N.size() != 14) return no("not a squeeze-and-excitation program");
  auto is = [&](int i, int op) { return N[i].op == op; };
  auto ew = [&](int i, int fn, std::vector<int> in) { return is(i, SOUFFLE_OP_ELEMENTWISE) && N[i].fn == fn && N[i].in == in; };
  const bool ok =
      is(0, SOUFFLE_OP_PLACEHOLDER) && !N[0].is_const && N[0].dtype == SOUFFLE_F32 && N[0].shape.size() == 2 &&
      is(1, SOUFFLE_OP_REDUCE) && N[1].fn == SOUFFLE_RED_MEAN && N[1].in[0] == 0 && N[1].axis == 0 && N[1].keepdim &&
      is(2, SOUFFLE_OP_PLACEHOLDER) && N[2].is_const && N[2].dtype == SOUFFLE_F32 &&
      is(3, SOUFFLE_OP_MATMUL) && N[3].a == 1 && N[3].b == 2 && N[3].trans_b && N[3].prec == SOUFFLE_F32 &&
      is(4, SOUFFLE_OP_PLACEHOLDER) && N[4].is_const && ew(5, SOUFFLE_EW_ADD, {3, 4}) &&
      ew(6, SOUFFLE_EW_SIGMOID, {5}) && ew(7, SOUFFLE_EW_MUL, {5, 6}) &&
      is(8, SOUFFLE_OP_PLACEHOLDER) && N[8].is_const && N[8].dtype == SOUFFLE_F32 &&
      is(9, SOUFFLE_OP_MATMUL) && N[9].a == 7 && N[9].b == 8 && N[9].trans_b && N[9].prec == SOUFFLE_F32 &&
      is(10, SOUFFLE_OP_PLACEHOLDER) && N[10].is_const && ew(11, SOUFFLE_EW_ADD, {9, 10}) &&
      ew(12, SOUFFLE_EW_SIGMOID, {11}) && ew(13, SOUFFLE_EW_MUL, {0, 12});
  if (!ok) return no("not a squeeze-and-excitation program");
  const int64_t HW = N[0].shape[0], C = N[0].shape[1], S = N[2].shape[0];
  if (N[2].shape != std::vector<int64_t>{S, C} || N[4].shape != std::vector<int64_t>{S} ||
      N[8].shape != std::vector<int64_t>{C, S} || N[10].shape != std::vector<int64_t>{C})
    return no("weight shapes");
  if (g.outputs.size() != 1 || g.outputs[0] != 13) return no("the only output must be the rescaled x");
  if (an.num_sp != 1) return no("the partition has more than one subprogram");
  if (C % 4 || C > 4096 || S > 4096) return no("channels must be a multiple of 4");
  // tile policy: channel blocks of <= 128 channels (a multiple of 4), row blocks to fill the SMs
  const int sms = dev.num_sms > 0 ? dev.num_sms : 148;
  int ncb = (int)((C + 127) / 128);
  while (ncb <= C / 4 && (C % ncb || (C / ncb) % 4)) ++ncb;
  if (ncb > C / 4) return no("no channel blocking");
  const int cbw = (int)(C / ncb);
  int nrb = std::max(1, std::min<int>((int)HW, sms / ncb));
  const int rows = (int)((HW + nrb - 1) / nrb);
  nrb = (int)((HW + rows - 1) / rows);
  if ((int64_t)rows * cbw > SE_MAX_TILE_FLOATS) return no("x tile exceeds shared memory");
  sp.x = 0; sp.W1 = 2; sp.b1 = 4; sp.W2 = 8; sp.b2 = 10; sp.y = 13;
  sp.HW = (int)HW; sp.C = (int)C; sp.S = (int)S;
  sp.nrb = nrb; sp.ncb = ncb; sp.rows = rows; sp.cbw = cbw;
  sp.reuse = flags == SOUFFLE_FLAG_NO_PREFETCH ? 0 : 1;
  int64_t o = 0;
  sp.o_ctrl = o; o = al(o + 256, 256);
  sp.o_part = o; o = al(o + 4LL * nrb * C, 256);
  sp.o_pooled = o; o = al(o + 4 * C, 256);
  sp.o_h = o; o = al(o + 4 * S, 256);
  sp.total = al(o, 4096);
  sp.on = true;
}

std::string se_describe(const SePlan& sp) {
  std::ostringstream os;
  if (!sp.on) {
    os << "pattern se: not used (" << sp.why_not << ")\n";
    return os.str();
  }
  os << "pattern se: squeeze-excitation HW=" << sp.HW << " C=" << sp.C << " S=" << sp.S
     << " -> 1 persistent launch (kernels/se.cu), " << sp.nrb * sp.ncb << " CTAs = " << sp.nrb << " row blocks x "
     << sp.ncb << " channel blocks of " << sp.rows << " x " << sp.cbw << ", 3 grid barriers, x "
     << (sp.reuse ? "reused from shared memory (Fig. 5(d))" : "re-read from global (Fig. 5(c))") << "\n";
  return os.str();
}

souffle_status se_run(Plan& p, void* ws, void* stream) {
  const SePlan& sp = p.se;
  auto ptr = [&](int node) -> void* { return p.buf_ptr[p.node_buf[node]]; };
  char* base = (char*)ws;
  SeParams prm{};
  prm.x = (const float*)ptr(sp.x);
  prm.W1 = (const float*)ptr(sp.W1);
  prm.b1 = (const float*)ptr(sp.b1);
  prm.W2 = (const float*)ptr(sp.W2);
  prm.b2 = (const float*)ptr(sp.b2);
  prm.y = (float*)ptr(sp.y);
  prm.part = (float*)(base + sp.o_part);
  prm.pooled = (float*)(base + sp.o_pooled);
  prm.h = (float*)(base + sp.o_h);
  prm.ctrl = (unsigned*)(base + sp.o_ctrl);
  prm.HW = sp.HW; prm.C = sp.C; prm.S = sp.S;
  prm.nrb = sp.nrb; prm.ncb = sp.ncb; prm.rows = sp.rows; prm.cbw = sp.cbw; prm.reuse = sp.reuse;
  if (((uintptr_t)prm.x | (uintptr_t)prm.y) & 15) return fail(SOUFFLE_E_INVALID_ARG, "x / y must be 16-byte aligned");
  cudaError_t e = se_launch(prm, sp.nrb * sp.ncb, (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("se launch: ") + cudaGetErrorString(e));
  return SOUFFLE_OK;
}

}  // namespace souffle
