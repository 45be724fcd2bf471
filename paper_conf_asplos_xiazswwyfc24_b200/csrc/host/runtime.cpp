// Execution runtime: workspace layout, program upload, TMA descriptor encoding, launches.
// One cooperative launch per subprogram (§4: "transforms each subprogram into
// a computation kernel"); every CUDA failure is reported as SOUFFLE_E_CUDA, there is no CPU path.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstring>
#include <stdexcept>
#include <string>

#include "../mmoe_types.h"
#include "plan.h"

namespace souffle {

extern thread_local std::string g_err;
souffle_status fail(souffle_status c, const std::string& m);

// kernels/exec.cu
cudaError_t exec_launch(const Params& prm, int grid, int smem, bool cooperative, cudaStream_t s);
cudaError_t exec_max_active(int smem, int* blocks_per_sm);

static int64_t al(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

souffle_status bert_init(Plan& p, void* ws, void* stream);
souffle_status bert_run(Plan& p, void* ws, void* stream);
souffle_status lstm_init(Plan& p, void* ws, void* stream);
souffle_status lstm_run(Plan& p, void* ws, void* stream);
souffle_status mmoe_run(Plan& p, void* ws, void* stream);
souffle_status swin_init(Plan& p, void* ws, void* stream);
souffle_status swin_run(Plan& p, void* ws, void* stream);
souffle_status se_run(Plan& p, void* ws, void* stream);
souffle_status mbconv_run(Plan& p, void* ws, void* stream);
souffle_status resnext_run(Plan& p, void* ws, void* stream);
souffle_status mmoe_init(Plan& p, void* ws, void* stream);

size_t workspace_bytes(Plan& p) {
  if (p.bert.on) return (size_t)p.bert.total;
  if (p.lstm.on) return (size_t)p.lstm.total;
  if (p.mmoe.on) return 2 * MMOE_SEG * 16;   // the parameter staging table
  if (p.swin.on) return (size_t)p.swin.total;
  if (p.se.on) return (size_t)p.se.total;
  if (p.mb.on) return (size_t)p.mb.total;
  if (p.rx.on) return (size_t)p.rx.total;
  WsLayout& w = p.ws;
  w.ctrl_off = 0;
  // barrier words + stage timestamps + 8 sub-stage marks per stage
  w.ctrl_bytes = al(256 + 8 * ((int64_t)p.stages.size() + 1) + 64 * (int64_t)p.stages.size() +
                        (p.profiling ? 8 * 4 * 160 * (int64_t)p.stages.size() : 0), 256) +
                 1024;   // + per-CTA progress words (watchdog diagnostics)
  int64_t o = w.ctrl_bytes;
  w.prog_off = o;
  int64_t q = 0;
  w.o_stages = q; q = al(q + (int64_t)p.stages.size() * sizeof(Stage), 256);
  w.o_members = q; q = al(q + (int64_t)p.members.size() * sizeof(GemmMember), 256);
  w.o_ins = q; q = al(q + (int64_t)p.ins.size() * sizeof(Ins), 256);
  w.o_addrs = q; q = al(q + (int64_t)p.addrs.size() * sizeof(Addr), 256);
  w.o_tabs = q; q = al(q + (int64_t)p.tabs.size() * sizeof(int32_t), 256);
  w.o_tmaps = q; q = al(q + (int64_t)p.tmaps.size() * 128, 256);
  w.o_zero = q; q = al(q + (int64_t)p.zero_list.size() * sizeof(int64_t), 256);
  w.prog_bytes = q;
  w.data_off = al(w.prog_off + w.prog_bytes, 4096);
  w.total = w.data_off + al(std::max<int64_t>(w.data_bytes, 256), 4096);
  return (size_t)w.total;
}

souffle_status query_device(int dev, souffle_device_desc* out) {
  cudaDeviceProp pr;
  cudaError_t e = cudaGetDeviceProperties(&pr, dev);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("cudaGetDeviceProperties: ") + cudaGetErrorString(e));
  std::memset(out, 0, sizeof(*out));
  out->num_sms = pr.multiProcessorCount;
  out->smem_per_sm = (int64_t)pr.sharedMemPerMultiprocessor;
  out->smem_per_block_max = (int64_t)pr.sharedMemPerBlockOptin;
  out->smem_reserved_per_block = (int64_t)pr.reservedSharedMemPerBlock;
  out->regs_per_sm = pr.regsPerMultiprocessor;
  out->max_threads_per_sm = pr.maxThreadsPerMultiProcessor;
  out->max_blocks_per_sm = pr.maxBlocksPerMultiProcessor;
  out->rule = 0;
  return SOUFFLE_OK;
}

typedef CUresult (*EncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiled get_encoder() {
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

static bool device_ok(std::string& why) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) { why = std::string("no CUDA device: ") + cudaGetErrorString(e); return false; }
  int maj = 0, mn = 0;
  cudaDeviceGetAttribute(&maj, cudaDevAttrComputeCapabilityMajor, dev);
  cudaDeviceGetAttribute(&mn, cudaDevAttrComputeCapabilityMinor, dev);
  if (maj != 10 || mn != 0) { why = "libsouffle kernels are built for sm_100a only (found sm_" + std::to_string(maj * 10 + mn) + ")"; return false; }
  return true;
}

souffle_status init_workspace(Plan& p, void* ws, void* stream) {
  std::string why;
  if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
  for (size_t s = 0; s < p.buf_ptr.size(); ++s)
    if (!p.buf_ptr[s]) return fail(SOUFFLE_E_STATE, "tensor " + std::to_string(p.buf_node[s]) + " is not bound");
  if (p.bert.on) return bert_init(p, ws, stream);
  if (p.lstm.on) return lstm_init(p, ws, stream);
  if (p.swin.on) return swin_init(p, ws, stream);
  if (p.se.on || p.mb.on || p.rx.on) {   // barrier counters start at zero (the last CTA of every launch resets them)
    cudaError_t e = cudaMemsetAsync(ws, 0, (size_t)(p.se.on ? p.se.total : p.mb.on ? p.mb.total : p.rx.total), (cudaStream_t)stream);
    if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("se workspace init: ") + cudaGetErrorString(e));
    p.inited_ws = ws;
    p.dirty = false;
    return SOUFFLE_OK;
  }
  if (p.mmoe.on) return mmoe_init(p, ws, stream);
  workspace_bytes(p);
  const WsLayout& w = p.ws;
  char* base = (char*)ws;
  char* data = base + w.data_off;
  // TMA descriptors (need final pointers)
  std::vector<uint8_t> tm(p.tmaps.size() * 128, 0);
  if (!p.tmaps.empty()) {
    EncodeTiled enc = get_encoder();
    if (!enc) return fail(SOUFFLE_E_CUDA, "cuTensorMapEncodeTiled unavailable");
    for (size_t i = 0; i < p.tmaps.size(); ++i) {
      const TmapSpec& t = p.tmaps[i];
      char* ptr = (t.buf >= 0 ? (char*)p.buf_ptr[t.buf] : data) + t.byte_off;
      CUtensorMap* m = (CUtensorMap*)&tm[i * 128];
      cuuint64_t dims[2] = {(cuuint64_t)t.cols, (cuuint64_t)t.rows};
      cuuint64_t strides[1] = {(cuuint64_t)t.cols * 2};
      cuuint32_t box[2] = {64, (cuuint32_t)t.box_rows};
      cuuint32_t es[2] = {1, 1};
      CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, ptr, dims, strides, box, es,
                       CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) return fail(SOUFFLE_E_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
    }
  }
  // pack the program region
  p.host_prog.assign((size_t)w.prog_bytes, 0);
  auto put = [&](int64_t off, const void* src, size_t n) { if (n) std::memcpy(&p.host_prog[off], src, n); };
  put(w.o_stages, p.stages.data(), p.stages.size() * sizeof(Stage));
  put(w.o_members, p.members.data(), p.members.size() * sizeof(GemmMember));
  put(w.o_ins, p.ins.data(), p.ins.size() * sizeof(Ins));
  {
    // resolve every address record to an absolute device pointer (no pointer-table lookups on device)
    std::vector<Addr> ra(p.addrs);
    for (Addr& a : ra) {
      char* b = a.buf >= 0 ? (char*)p.buf_ptr[a.buf] : data;
      a.ptr = (uint64_t)(b + a.base * (a.dtype == 1 ? 2 : 4));
    }
    put(w.o_addrs, ra.data(), ra.size() * sizeof(Addr));
  }
  put(w.o_tabs, p.tabs.data(), p.tabs.size() * sizeof(int32_t));
  put(w.o_tmaps, tm.data(), tm.size());
  put(w.o_zero, p.zero_list.data(), p.zero_list.size() * sizeof(int64_t));
  cudaStream_t s = (cudaStream_t)stream;
  cudaError_t e = cudaMemsetAsync(base, 0, (size_t)w.ctrl_bytes, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(base + w.prog_off, p.host_prog.data(), (size_t)w.prog_bytes,
                                            cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemsetAsync(data, 0, (size_t)(w.total - w.data_off), s);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("workspace init: ") + cudaGetErrorString(e));
  p.inited_ws = ws;
  p.dirty = false;
  return SOUFFLE_OK;
}

souffle_status run_plan(Plan& p, void* ws, void* stream) {
  if (p.dirty || p.inited_ws != ws)
    return fail(SOUFFLE_E_STATE, "call souffle_workspace_init after binding (bindings or workspace changed)");
  if (p.bert.on) {
    std::string why;
    if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
    return bert_run(p, ws, stream);
  }
  if (p.lstm.on) {
    std::string why;
    if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
    return lstm_run(p, ws, stream);
  }
  if (p.mmoe.on) {
    std::string why;
    if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
    return mmoe_run(p, ws, stream);
  }
  if (p.swin.on) {
    std::string why;
    if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
    return swin_run(p, ws, stream);
  }
  if (p.se.on) {
    std::string why;
    if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
    return se_run(p, ws, stream);
  }
  if (p.mb.on) {
    std::string why;
    if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
    return mbconv_run(p, ws, stream);
  }
  if (p.rx.on) {
    std::string why;
    if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
    return resnext_run(p, ws, stream);
  }
  static int max_active = -1;
  if (max_active < 0) {
    std::string why;
    if (!device_ok(why)) return fail(SOUFFLE_E_UNSUPPORTED, why);
    int b = 0;
    cudaError_t e = exec_max_active(EXEC_SMEM, &b);
    if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("occupancy query: ") + cudaGetErrorString(e));
    max_active = b;
  }
  int dev = 0, nsm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const WsLayout& w = p.ws;
  char* base = (char*)ws;
  Params prm;
  std::memset(&prm, 0, sizeof(prm));
  prm.stages = (const Stage*)(base + w.prog_off + w.o_stages);
  prm.members = (const GemmMember*)(base + w.prog_off + w.o_members);
  prm.ins = (const Ins*)(base + w.prog_off + w.o_ins);
  prm.addrs = (const Addr*)(base + w.prog_off + w.o_addrs);
  prm.tabs = (const int32_t*)(base + w.prog_off + w.o_tabs);
  prm.tmaps = (const void*)(base + w.prog_off + w.o_tmaps);
  prm.zero_list = (const int64_t*)(base + w.prog_off + w.o_zero);
  prm.n_zero = (int32_t)(p.zero_list.size() / 2);
  prm.ws_data = base + w.data_off;
  prm.ctrl = (unsigned int*)(base + w.ctrl_off);
  prm.prof = p.profiling ? (unsigned long long*)(base + w.ctrl_off + 256) : nullptr;
  prm.progress = (unsigned int*)(base + w.ctrl_off + w.ctrl_bytes - 1024);
  prm.n_stages_total = (int32_t)p.stages.size();
  for (size_t i = 0; i < p.buf_ptr.size(); ++i) prm.bufs[i] = p.buf_ptr[i];
  cudaStream_t s = (cudaStream_t)stream;
  for (const Launch& L : p.launches) {
    int grid = L.grid;
    if (L.cooperative) {
      int cap = max_active * nsm;
      if (cap < 1) return fail(SOUFFLE_E_RESOURCE, "persistent kernel cannot be resident");
      if (grid > cap) grid = cap;  // persistent stages loop over their tasks
    }
    // the tensor cache's slot placement assumes the planned grid (one CTA per SM)
    if (L.smem > EXEC_SMEM && grid != L.grid)
      return fail(SOUFFLE_E_RESOURCE, "tensor-cache launch needs its planned grid (plan made for another device?)");
    prm.first = L.first;
    prm.count = L.count;
    prm.cooperative = L.cooperative;
    prm.uses_tc = L.uses_tc;
    prm.is_last = L.is_last;
    cudaError_t e = exec_launch(prm, grid, L.smem, L.cooperative != 0, s);
    if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("launch: ") + cudaGetErrorString(e));
  }
  return SOUFFLE_OK;
}

souffle_status read_profile_raw(Plan& p, void* ws, unsigned long long* out, int cap, int* n) {
  if (p.lstm.on) {   // [T][4] timestamps of the profiled CTA: step start, operands in smem, gates, -
    const size_t cnt = 4 * (size_t)p.lstm.T;
    if ((size_t)cap < cnt) return fail(SOUFFLE_E_INVALID_ARG, "profile buffer too small");
    cudaError_t e = cudaDeviceSynchronize();
    if (e == cudaSuccess) e = cudaMemcpy(out, (char*)ws + p.lstm.o_prof, cnt * 8, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("profile read: ") + cudaGetErrorString(e));
    *n = (int)cnt;
    return SOUFFLE_OK;
  }
  if (p.bert.on) {   // [0, ns): stage starts, ns+1: end; then 16 sub-stage marks per stage
    const size_t cnt = 17 * (size_t)p.bert.nstages + 2;
    if ((size_t)cap < cnt) return fail(SOUFFLE_E_INVALID_ARG, "profile buffer too small");
    cudaError_t e = cudaDeviceSynchronize();
    if (e == cudaSuccess) e = cudaMemcpy(out, (char*)ws + p.bert.o_prof, cnt * 8, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("profile read: ") + cudaGetErrorString(e));
    *n = (int)cnt;
    return SOUFFLE_OK;
  }
  size_t cnt = p.stages.size() + 1 + 8 * p.stages.size() + (p.profiling ? 4 * 160 * p.stages.size() : 0);
  if ((size_t)cap < cnt) return fail(SOUFFLE_E_INVALID_ARG, "profile buffer too small");
  cudaError_t e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(out, (char*)ws + p.ws.ctrl_off + 256, cnt * 8, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("profile read: ") + cudaGetErrorString(e));
  *n = (int)cnt;
  return SOUFFLE_OK;
}

souffle_status read_profile(Plan& p, void* ws, double* us, int cap, int* n) {
  if (p.bert.on) {
    const int ns = p.bert.nstages;
    std::vector<unsigned long long> t(ns + 2, 0);
    cudaError_t e = cudaDeviceSynchronize();
    if (e == cudaSuccess) e = cudaMemcpy(t.data(), (char*)ws + p.bert.o_prof, t.size() * 8, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("profile read: ") + cudaGetErrorString(e));
    int k = 0;
    for (int s = 0; s < ns && k < cap; ++s, ++k) {
      unsigned long long nx = s + 1 < ns ? t[s + 1] : t[ns + 1];
      us[k] = nx > t[s] ? (double)(nx - t[s]) * 1e-3 : -1.0;
    }
    *n = k;
    return SOUFFLE_OK;
  }
  std::vector<unsigned long long> t(p.stages.size() + 1, 0);
  cudaError_t e = cudaDeviceSynchronize();
  if (e == cudaSuccess)
    e = cudaMemcpy(t.data(), (char*)ws + p.ws.ctrl_off + 256, t.size() * 8, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return fail(SOUFFLE_E_CUDA, std::string("profile read: ") + cudaGetErrorString(e));
  // duration of stage s = next timestamp in its launch (stage start or launch end) - its start
  int k = 0;
  for (const Launch& L : p.launches)
    for (int s = L.first; s < L.first + L.count && k < cap; ++s, ++k) {
      unsigned long long nx = (s + 1 < L.first + L.count) ? t[s + 1] : t[L.first + L.count];
      us[k] = (nx > t[s]) ? (double)(nx - t[s]) * 1e-3 : -1.0;
    }
  *n = k;
  return SOUFFLE_OK;
}

}  // namespace souffle
