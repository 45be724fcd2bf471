// extern "C" entry points of libsouffle (declared and documented in include/souffle.h).
#include <algorithm>
#include <cstring>
#include <exception>
#include <new>
#include <stdexcept>
#include <string>

#include "plan.h"

struct souffle_graph_s {
  souffle::Graph g;
};
struct souffle_plan_s {
  souffle::Plan p;
};

namespace souffle {
thread_local std::string g_err;

struct Error : std::runtime_error {
  souffle_status code;
  Error(souffle_status c, const std::string& m) : std::runtime_error(m), code(c) {}
};

souffle_status fail(souffle_status c, const std::string& m) {
  g_err = m;
  return c;
}

template <class F>
souffle_status guard(F&& f) {
  g_err.clear();
  try {
    f();
    return SOUFFLE_OK;
  } catch (const Error& e) {
    return fail(e.code, e.what());
  } catch (const std::bad_alloc&) {
    return fail(SOUFFLE_E_OOM, "host allocation failed");
  } catch (const std::exception& e) {
    return fail(SOUFFLE_E_INVALID_ARG, e.what());
  }
}

static void need(bool c, souffle_status code, const std::string& m) {
  if (!c) throw Error(code, m);
}

static Graph& G(souffle_graph g) {
  need(g != nullptr, SOUFFLE_E_INVALID_ARG, "null graph");
  return g->g;
}
static Plan& PL(souffle_plan p) {
  need(p != nullptr, SOUFFLE_E_INVALID_ARG, "null plan");
  return p->p;
}
static void check_t(const Graph& g, souffle_tensor t) {
  need(t >= 0 && t < (int)g.nodes.size(), SOUFFLE_E_INVALID_ARG, "tensor id out of range: " + std::to_string(t));
}
static int push(Graph& g, Node n) {
  g.nodes.push_back(std::move(n));
  return (int)g.nodes.size() - 1;
}

// runtime.cpp
souffle_status run_plan(Plan& p, void* ws, void* stream);
souffle_status init_workspace(Plan& p, void* ws, void* stream);
souffle_status query_device(int dev, souffle_device_desc* out);
size_t workspace_bytes(Plan& p);
souffle_status read_profile(Plan& p, void* ws, double* us, int cap, int* n);
souffle_status read_profile_raw(Plan& p, void* ws, unsigned long long* out, int cap, int* n);

}  // namespace souffle

using namespace souffle;

extern "C" {

const char* souffle_last_error(void) { return g_err.c_str(); }
const char* souffle_version(void) { return "souffle-b200 0.1 (sm_100a)"; }

souffle_status souffle_graph_create(souffle_graph* out) {
  return guard([&] {
    need(out != nullptr, SOUFFLE_E_INVALID_ARG, "null out");
    *out = new souffle_graph_s();
  });
}

souffle_status souffle_graph_destroy(souffle_graph g) {
  delete g;
  g_err.clear();
  return SOUFFLE_OK;
}

souffle_status souffle_placeholder(souffle_graph g, int32_t ndim, const int64_t* shape, int32_t dtype,
                                   int32_t is_constant, souffle_tensor* out) {
  return guard([&] {
    Graph& gr = G(g);
    need(out && shape && ndim >= 1 && ndim <= 8, SOUFFLE_E_INVALID_ARG, "bad placeholder arguments");
    need(dtype == SOUFFLE_F32 || dtype == SOUFFLE_BF16, SOUFFLE_E_INVALID_ARG, "bad dtype");
    Node n;
    n.op = SOUFFLE_OP_PLACEHOLDER;
    n.shape.assign(shape, shape + ndim);
    for (auto d : n.shape) need(d > 0, SOUFFLE_E_SHAPE, "non-positive dim");
    n.dtype = dtype;
    n.is_const = is_constant ? 1 : 0;
    *out = push(gr, n);
  });
}

souffle_status souffle_matmul(souffle_graph g, souffle_tensor a, souffle_tensor b, int32_t trans_b,
                              int32_t precision, souffle_tensor* out) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, a);
    check_t(gr, b);
    need(out != nullptr, SOUFFLE_E_INVALID_ARG, "null out");
    need(precision == SOUFFLE_F32 || precision == SOUFFLE_BF16, SOUFFLE_E_INVALID_ARG, "bad precision");
    const auto& as = gr.nodes[a].shape;
    const auto& bs = gr.nodes[b].shape;
    need(as.size() >= 2 && bs.size() >= 2, SOUFFLE_E_SHAPE, "matmul operands need >= 2 dims");
    int64_t K = as.back();
    int64_t Kb = trans_b ? bs.back() : bs[bs.size() - 2];
    int64_t N = trans_b ? bs[bs.size() - 2] : bs.back();
    need(K == Kb, SOUFFLE_E_SHAPE, "matmul reduce extents differ");
    need(bs.size() == 2 || (bs.size() == as.size() && std::equal(as.begin(), as.end() - 2, bs.begin())),
         SOUFFLE_E_SHAPE, "matmul batch dims differ");
    Node n;
    n.op = SOUFFLE_OP_MATMUL;
    n.a = a;
    n.b = b;
    n.trans_b = trans_b ? 1 : 0;
    n.prec = precision;
    n.shape.assign(as.begin(), as.end() - 1);
    n.shape.push_back(N);
    *out = push(gr, n);
  });
}

souffle_status souffle_elementwise(souffle_graph g, int32_t op, int32_t n_in, const souffle_tensor* in,
                                   double scalar, souffle_tensor* out) {
  return guard([&] {
    Graph& gr = G(g);
    need(out && in, SOUFFLE_E_INVALID_ARG, "null argument");
    need(op >= SOUFFLE_EW_ADD && op <= SOUFFLE_EW_MUL_SCALAR, SOUFFLE_E_INVALID_ARG, "bad elementwise op");
    int want = op <= SOUFFLE_EW_MAX ? 2 : 1;
    need(n_in == want, SOUFFLE_E_INVALID_ARG, "wrong number of inputs");
    Node n;
    n.op = SOUFFLE_OP_ELEMENTWISE;
    n.fn = op;
    n.scalar = scalar;
    size_t nd = 0;
    for (int k = 0; k < n_in; ++k) {
      check_t(gr, in[k]);
      n.in.push_back(in[k]);
      nd = std::max(nd, gr.nodes[in[k]].shape.size());
    }
    n.shape.assign(nd, 1);
    for (size_t d = 0; d < nd; ++d) {
      int64_t m = 1;
      for (int k = 0; k < n_in; ++k) {
        const auto& s = gr.nodes[in[k]].shape;
        int off = (int)nd - (int)s.size();
        if ((int)d - off < 0) continue;
        int64_t x = s[d - off];
        need(x == 1 || m == 1 || x == m, SOUFFLE_E_SHAPE, "shapes not broadcastable");
        m = std::max(m, x);
      }
      n.shape[d] = m;
    }
    *out = push(gr, n);
  });
}

souffle_status souffle_reduce(souffle_graph g, int32_t op, souffle_tensor in, int32_t axis, int32_t keepdim,
                              souffle_tensor* out) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, in);
    need(out != nullptr, SOUFFLE_E_INVALID_ARG, "null out");
    need(op >= SOUFFLE_RED_SUM && op <= SOUFFLE_RED_MEAN, SOUFFLE_E_INVALID_ARG, "bad reduce op");
    const auto& s = gr.nodes[in].shape;
    int ax = axis < 0 ? axis + (int)s.size() : axis;
    need(ax >= 0 && ax < (int)s.size(), SOUFFLE_E_SHAPE, "bad axis");
    Node n;
    n.op = SOUFFLE_OP_REDUCE;
    n.fn = op;
    n.in = {in};
    n.axis = ax;
    n.keepdim = keepdim ? 1 : 0;
    n.shape = s;
    if (keepdim) n.shape[ax] = 1; else n.shape.erase(n.shape.begin() + ax);
    if (n.shape.empty()) n.shape.push_back(1);
    *out = push(gr, n);
  });
}

souffle_status souffle_reshape(souffle_graph g, souffle_tensor in, int32_t ndim, const int64_t* shape,
                               souffle_tensor* out) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, in);
    need(out && shape && ndim >= 1 && ndim <= 8, SOUFFLE_E_INVALID_ARG, "bad reshape arguments");
    Node n;
    n.op = SOUFFLE_OP_RESHAPE;
    n.in = {in};
    n.shape.assign(shape, shape + ndim);
    need(numel(n.shape) == numel(gr.nodes[in].shape), SOUFFLE_E_SHAPE, "reshape changes the element count");
    *out = push(gr, n);
  });
}

souffle_status souffle_permute(souffle_graph g, souffle_tensor in, const int32_t* perm, souffle_tensor* out) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, in);
    need(out && perm, SOUFFLE_E_INVALID_ARG, "null argument");
    const auto& s = gr.nodes[in].shape;
    Node n;
    n.op = SOUFFLE_OP_PERMUTE;
    n.in = {in};
    std::vector<int> seen(s.size(), 0);
    for (size_t k = 0; k < s.size(); ++k) {
      need(perm[k] >= 0 && perm[k] < (int)s.size() && !seen[perm[k]], SOUFFLE_E_INVALID_ARG, "bad permutation");
      seen[perm[k]] = 1;
      n.perm.push_back(perm[k]);
      n.shape.push_back(s[perm[k]]);
    }
    *out = push(gr, n);
  });
}

souffle_status souffle_slice(souffle_graph g, souffle_tensor in, const int64_t* begin, const int64_t* end,
                             const int64_t* stride, souffle_tensor* out) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, in);
    need(out && begin && end && stride, SOUFFLE_E_INVALID_ARG, "null argument");
    const auto& s = gr.nodes[in].shape;
    Node n;
    n.op = SOUFFLE_OP_SLICE;
    n.in = {in};
    for (size_t d = 0; d < s.size(); ++d) {
      need(stride[d] > 0 && begin[d] >= 0 && end[d] <= s[d] && begin[d] < end[d], SOUFFLE_E_SHAPE, "bad slice");
      n.begin.push_back(begin[d]);
      n.end.push_back(end[d]);
      n.stride.push_back(stride[d]);
      n.shape.push_back((end[d] - begin[d] + stride[d] - 1) / stride[d]);
    }
    *out = push(gr, n);
  });
}

souffle_status souffle_roll(souffle_graph g, souffle_tensor in, const int64_t* shifts, souffle_tensor* out) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, in);
    need(out && shifts, SOUFFLE_E_INVALID_ARG, "null argument");
    const auto& s = gr.nodes[in].shape;
    Node n;
    n.op = SOUFFLE_OP_ROLL;
    n.in = {in};
    n.shape = s;
    for (size_t d = 0; d < s.size(); ++d) n.shifts.push_back(((shifts[d] % s[d]) + s[d]) % s[d]);
    *out = push(gr, n);
  });
}

souffle_status souffle_mark_output(souffle_graph g, souffle_tensor t) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, t);
    need(gr.nodes[t].op != SOUFFLE_OP_PLACEHOLDER, SOUFFLE_E_INVALID_ARG, "a placeholder cannot be an output");
    if (std::find(gr.outputs.begin(), gr.outputs.end(), t) == gr.outputs.end()) gr.outputs.push_back(t);
  });
}

souffle_status souffle_graph_num_nodes(souffle_graph g, int32_t* n) {
  return guard([&] {
    need(n != nullptr, SOUFFLE_E_INVALID_ARG, "null out");
    *n = (int32_t)G(g).nodes.size();
  });
}

souffle_status souffle_graph_node(souffle_graph g, souffle_tensor t, int32_t* op, int32_t* ndim, int64_t* shape,
                                  int32_t* dtype) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, t);
    const Node& n = gr.nodes[t];
    if (op) *op = n.op;
    if (ndim) *ndim = (int32_t)n.shape.size();
    if (shape) std::copy(n.shape.begin(), n.shape.end(), shape);
    if (dtype) *dtype = n.op == SOUFFLE_OP_PLACEHOLDER ? n.dtype : SOUFFLE_F32;
  });
}

souffle_status souffle_set_te_resources(souffle_graph g, souffle_tensor te, int64_t grid, int64_t smem, int32_t regs,
                                        int32_t threads) {
  return guard([&] {
    Graph& gr = G(g);
    check_t(gr, te);
    Node& n = gr.nodes[te];
    need(n.op != SOUFFLE_OP_PLACEHOLDER, SOUFFLE_E_INVALID_ARG, "placeholders have no resources");
    need(grid >= 0 && smem >= 0 && regs >= 0 && threads >= 0, SOUFFLE_E_INVALID_ARG, "negative resource");
    n.res_override = true;
    n.r_grid = grid;
    n.r_smem = smem;
    n.r_regs = regs;
    n.r_threads = threads;
  });
}

souffle_status souffle_device_query(int32_t cuda_device, souffle_device_desc* out) {
  g_err.clear();
  if (!out) return fail(SOUFFLE_E_INVALID_ARG, "null out");
  return query_device(cuda_device, out);
}

souffle_status souffle_device_b200(souffle_device_desc* out) {
  return guard([&] {
    need(out != nullptr, SOUFFLE_E_INVALID_ARG, "null out");
    std::memset(out, 0, sizeof(*out));
    out->num_sms = 148;
    out->smem_per_sm = 233472;
    out->smem_per_block_max = 232448;
    out->smem_reserved_per_block = 1024;
    out->regs_per_sm = 65536;
    out->max_threads_per_sm = 2048;
    out->max_blocks_per_sm = 32;
    out->rule = 0;
    out->capacity_C = 0;
  });
}

souffle_status souffle_partition(souffle_graph g, const souffle_device_desc* dev, uint32_t flags, souffle_plan* out) {
  return guard([&] {
    Graph& gr = G(g);
    need(dev && out, SOUFFLE_E_INVALID_ARG, "null argument");
    need(!gr.outputs.empty(), SOUFFLE_E_STATE, "graph has no outputs (souffle_mark_output)");
    need(dev->rule == 0 || dev->rule == 1, SOUFFLE_E_INVALID_ARG, "bad rule");
    auto* pl = new souffle_plan_s();
    try {
      pl->p.g = gr;
      pl->p.dev = *dev;
      pl->p.flags = flags;
      analyse(pl->p.g, *dev, pl->p.an);
      lower(pl->p);
      workspace_bytes(pl->p);
    } catch (...) {
      delete pl;
      throw;
    }
    *out = pl;
  });
}

souffle_status souffle_plan_destroy(souffle_plan p) {
  delete p;
  g_err.clear();
  return SOUFFLE_OK;
}

souffle_status souffle_plan_num_nodes(souffle_plan p, int32_t* n) {
  return guard([&] { need(n, SOUFFLE_E_INVALID_ARG, "null out"); *n = (int32_t)PL(p).g.nodes.size(); });
}
souffle_status souffle_plan_num_tes(souffle_plan p, int32_t* n) {
  return guard([&] { need(n, SOUFFLE_E_INVALID_ARG, "null out"); *n = (int32_t)PL(p).an.order.size(); });
}
souffle_status souffle_plan_num_subprograms(souffle_plan p, int32_t* n) {
  return guard([&] { need(n, SOUFFLE_E_INVALID_ARG, "null out"); *n = PL(p).an.num_sp; });
}
souffle_status souffle_plan_assignment(souffle_plan p, int32_t* te_to_sp) {
  return guard([&] {
    need(te_to_sp, SOUFFLE_E_INVALID_ARG, "null out");
    const auto& a = PL(p).an.assign;
    std::copy(a.begin(), a.end(), te_to_sp);
  });
}
souffle_status souffle_plan_bfs_order(souffle_plan p, int32_t* order) {
  return guard([&] {
    need(order, SOUFFLE_E_INVALID_ARG, "null out");
    const auto& o = PL(p).an.order;
    std::copy(o.begin(), o.end(), order);
  });
}
souffle_status souffle_plan_te_info(souffle_plan p, souffle_tensor te, int32_t* dep_kind, int32_t* intensity,
                                    int64_t* ops, int64_t* accesses, int64_t* grid, int64_t* smem, int32_t* regs,
                                    int32_t* threads) {
  return guard([&] {
    Plan& P = PL(p);
    check_t(P.g, te);
    const Analysis& a = P.an;
    if (dep_kind) *dep_kind = a.dep[te];
    if (intensity) *intensity = a.ci[te];
    if (ops) *ops = a.ops[te];
    if (accesses) *accesses = a.acc[te];
    Resources r = a.res[te];
    if (grid) *grid = r.grid;
    if (smem) *smem = r.smem;
    if (regs) *regs = r.regs;
    if (threads) *threads = r.threads;
  });
}
souffle_status souffle_plan_reuse_set(souffle_plan p, souffle_tensor t, int32_t* consumers, int32_t cap, int32_t* n,
                                      int32_t* kind) {
  return guard([&] {
    Plan& P = PL(p);
    check_t(P.g, t);
    const auto& cs = P.an.cons[t];
    if (n) *n = (int32_t)cs.size();
    if (kind) *kind = P.an.reuse_kind[t];
    if (consumers)
      for (int k = 0; k < (int)cs.size() && k < cap; ++k) consumers[k] = cs[k];
  });
}
souffle_status souffle_plan_index_map(souffle_plan p, souffle_tensor fused_out, souffle_tensor source,
                                      int64_t* src_offset) {
  return guard([&] {
    Plan& P = PL(p);
    check_t(P.g, fused_out);
    check_t(P.g, source);
    need(src_offset, SOUFFLE_E_INVALID_ARG, "null out");
    std::vector<int64_t> m;
    need(index_map(P.g, fused_out, source, m), SOUFFLE_E_INVALID_ARG, "no one-relies-on-one path");
    std::copy(m.begin(), m.end(), src_offset);
  });
}
souffle_status souffle_plan_hgroup(souffle_plan p, souffle_tensor te, int32_t* level, int32_t* group, int32_t* kind) {
  return guard([&] {
    Plan& P = PL(p);
    check_t(P.g, te);
    if (level) *level = P.an.level[te];
    int gid = P.an.hgid[te];
    if (group) *group = gid;
    if (kind) *kind = gid >= 0 ? P.an.hkind[gid] : -1;
  });
}
souffle_status souffle_plan_debug_region(souffle_plan p, const char* name, int64_t* offset, int64_t* bytes) {
  return guard([&] {
    Plan& P = PL(p);
    if (!name || !offset || !bytes) throw Error(SOUFFLE_E_INVALID_ARG, "null argument");
    const BertPlan& b = P.bert;
    if (P.swin.on && std::string(name) == "trace") {   // Swin debug trace: one u64 stamp per launch
      *offset = P.swin.o_trace;
      *bytes = 8 * (int64_t)P.swin.launches;
      return;
    }
    if (!b.on) throw Error(SOUFFLE_E_UNSUPPORTED, "the plan does not use the BERT pattern kernel");
    const int64_t S = b.S, H = b.H, F = b.F;
    const std::string n(name);
    if (n == "xb") { *offset = b.o_xb; *bytes = S * H * 2; }
    else if (n == "l1b") { *offset = b.o_l1b; *bytes = S * H * 2; }
    else if (n == "l1f") { *offset = b.o_l1f; *bytes = S * H * 4; }
    else if (n == "xf") { *offset = b.o_xf; *bytes = S * H * 4; }
    else if (n == "qk") { *offset = b.o_qk; *bytes = 2 * S * H * 2; }
    else if (n == "vt") { *offset = b.o_vt; *bytes = S * H * 2; }
    else if (n == "h") { *offset = b.o_h; *bytes = S * F * 2; }
    else if (n == "part_o") { *offset = b.o_part_o; *bytes = (int64_t)b.out.nsplit * S * H * 4; }
    else if (n == "part_2") { *offset = b.o_part_2; *bytes = (int64_t)b.ffn2.nsplit * S * H * 4; }
    else throw Error(SOUFFLE_E_INVALID_ARG, "unknown debug region " + n);
  });
}

souffle_status souffle_plan_exec_info(souffle_plan p, int32_t* launches, int32_t* stages, int32_t* barriers) {
  return guard([&] {
    Plan& P = PL(p);
    if (P.mmoe.on) {
      if (launches) *launches = 1;
      if (stages) *stages = 5;
      if (barriers) *barriers = 0;
      return;
    }
    if (P.lstm.on) {
      if (launches) *launches = 1;
      if (stages) *stages = P.lstm.L + P.lstm.T - 1;   // wavefront steps
      if (barriers) *barriers = 0;                      // point-to-point flags only
      return;
    }
    if (P.bert.on) {
      if (launches) *launches = 1;
      if (stages) *stages = P.bert.nstages;
      if (barriers) *barriers = P.bert.nstages - 1;
      return;
    }
    if (P.se.on) {
      if (launches) *launches = 1;
      if (stages) *stages = 4;
      if (barriers) *barriers = 3;
      return;
    }
    if (P.mb.on) {   // expand | depthwise + pool | fc1 | gates + project (+ split-K finish)
      if (launches) *launches = 1;
      if (stages) *stages = 4;
      if (barriers) *barriers = 3;
      return;
    }
    if (P.rx.on) {   // 1x1 (+ projection) | grouped 3x3 | 1x1 + shortcut
      if (launches) *launches = 1;
      if (stages) *stages = 3;
      if (barriers) *barriers = 2;
      return;
    }
    if (P.swin.on) {   // one kernel per fused subprogram, replayed as one CUDA graph
      if (launches) *launches = P.swin.launches;
      if (stages) *stages = P.swin.launches;
      if (barriers) *barriers = 0;
      return;
    }
    if (launches) *launches = (int32_t)P.launches.size();
    if (stages) *stages = (int32_t)P.stages.size();
    if (barriers) *barriers = P.n_barriers;
  });
}
souffle_status souffle_plan_describe(souffle_plan p, const char** text) {
  return guard([&] {
    need(text, SOUFFLE_E_INVALID_ARG, "null out");
    *text = PL(p).text.c_str();
  });
}
souffle_status souffle_plan_workspace_bytes(souffle_plan p, size_t* bytes) {
  return guard([&] {
    need(bytes, SOUFFLE_E_INVALID_ARG, "null out");
    *bytes = workspace_bytes(PL(p));
  });
}
souffle_status souffle_bind(souffle_plan p, souffle_tensor t, void* device_ptr) {
  return guard([&] {
    Plan& P = PL(p);
    check_t(P.g, t);
    need(device_ptr != nullptr, SOUFFLE_E_INVALID_ARG, "null device pointer");
    int slot = P.node_buf[t];
    need(slot >= 0, SOUFFLE_E_INVALID_ARG, "tensor is neither a placeholder nor an output");
    if (P.buf_ptr[slot] != device_ptr) P.dirty = true;
    P.buf_ptr[slot] = device_ptr;
  });
}
souffle_status souffle_workspace_init(souffle_plan p, void* workspace, void* stream) {
  g_err.clear();
  if (!p || !workspace) return fail(SOUFFLE_E_INVALID_ARG, "null argument");
  try {
    return init_workspace(p->p, workspace, stream);
  } catch (const std::exception& e) {
    return fail(SOUFFLE_E_INVALID_ARG, e.what());
  }
}
souffle_status souffle_run(souffle_plan p, void* workspace, void* stream) {
  g_err.clear();
  if (!p || !workspace) return fail(SOUFFLE_E_INVALID_ARG, "null argument");
  return run_plan(p->p, workspace, stream);
}

souffle_status souffle_plan_set_profiling(souffle_plan p, int32_t on) {
  // the control region's size depends on the flag (runtime.cpp workspace_bytes): a change requires
  // souffle_plan_workspace_bytes + souffle_workspace_init again, so mark the plan dirty
  return guard([&] {
    Plan& P = PL(p);
    if (P.profiling != (on != 0)) P.dirty = true;
    P.profiling = on != 0;
  });
}
souffle_status souffle_plan_read_profile(souffle_plan p, void* workspace, double* stage_us, int32_t cap, int32_t* n) {
  g_err.clear();
  if (!p || !workspace || !stage_us || !n) return fail(SOUFFLE_E_INVALID_ARG, "null argument");
  return read_profile(p->p, workspace, stage_us, cap, n);
}
souffle_status souffle_plan_read_profile_raw(souffle_plan p, void* workspace, uint64_t* stamps, int32_t cap,
                                             int32_t* n) {
  g_err.clear();
  if (!p || !workspace || !stamps || !n) return fail(SOUFFLE_E_INVALID_ARG, "null argument");
  return read_profile_raw(p->p, workspace, (unsigned long long*)stamps, cap, n);
}

}  // extern "C"
