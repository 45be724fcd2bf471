// Global computation-graph analysis and resource-aware partitioning (§5, Alg. 1).
//
//   classify      §5.2: one-relies-on-one (no reduce axis) vs one-relies-on-many.
//                 §5.3: ratio = arithmetic ops / memory accesses, < 3 -> memory-intensive.
//   reuse sets    §5.1: s(t) = consumers of t; spatial if independent, else temporal.
//   order         Alg. 1 line 2 "BFS(P)" (L1258); reading R3: Kahn's algorithm, FIFO queue.
//   partition     §5.4 L998-1012 + Alg. 1 lines 2-9: greedy; only CI TEs open subprograms.
//   hgroups       §6.1 L1062-1084 horizontal transformation candidates (reading R8).
// Every result here is integer-valued and must equal oracle/analysis.py bit-exactly.
#include <algorithm>
#include <cstring>
#include <deque>
#include <stdexcept>

#include "ir.h"

namespace souffle {

int64_t numel(const std::vector<int64_t>& s) {
  int64_t n = 1;
  for (auto d : s) n *= d;
  return n;
}

std::vector<int> node_inputs(const Node& n) {
  switch (n.op) {
    case SOUFFLE_OP_PLACEHOLDER: return {};
    case SOUFFLE_OP_MATMUL: return {n.a, n.b};
    default: return n.in;
  }
}

std::vector<int> distinct_inputs(const Node& n) {
  auto v = node_inputs(n);
  std::sort(v.begin(), v.end());
  v.erase(std::unique(v.begin(), v.end()), v.end());
  return v;
}

bool is_or_op(int op) {
  return op == SOUFFLE_OP_ELEMENTWISE || op == SOUFFLE_OP_RESHAPE || op == SOUFFLE_OP_PERMUTE ||
         op == SOUFFLE_OP_SLICE || op == SOUFFLE_OP_ROLL;
}
bool is_mr_op(int op) { return op == SOUFFLE_OP_MATMUL || op == SOUFFLE_OP_REDUCE; }

static int occupancy(const souffle_device_desc& d, const Resources& r) {
  int64_t lim = d.max_blocks_per_sm;
  if (r.smem > 0) lim = std::min<int64_t>(lim, d.smem_per_sm / (r.smem + d.smem_reserved_per_block));
  if ((int64_t)r.regs * r.threads > 0) lim = std::min<int64_t>(lim, d.regs_per_sm / ((int64_t)r.regs * r.threads));
  if (r.threads > 0) lim = std::min<int64_t>(lim, d.max_threads_per_sm / r.threads);
  return (int)lim;
}

// rule 1: paper's analytical model max_grid * max_occ <= C (shared-memory bytes; '<=' per Fig. 2).
// rule 0: B200-exact co-residency for a cooperative launch.
bool fits(const souffle_device_desc& d, const Resources& r) {
  if (d.rule == 1) return r.grid * r.smem <= d.capacity_C;
  return r.grid <= (int64_t)d.num_sms * occupancy(d, r);
}

void analyse(const Graph& g, const souffle_device_desc& dev, Analysis& a) {
  const int n = (int)g.nodes.size();
  a.n = n;
  a.dep.assign(n, -1);
  a.ci.assign(n, 0);
  a.ops.assign(n, 0);
  a.acc.assign(n, 0);
  a.cons.assign(n, {});
  a.reuse_kind.assign(n, -1);
  a.level.assign(n, -1);
  a.res.assign(n, Resources{});
  a.assign.assign(n, -1);
  a.hgid.assign(n, -1);
  a.hkind.clear();
  a.order.clear();

  // ---- classification (§5.2, §5.3)
  for (int i = 0; i < n; ++i) {
    const Node& nd = g.nodes[i];
    if (nd.op == SOUFFLE_OP_PLACEHOLDER) continue;
    int64_t O = numel(nd.shape);
    int64_t ops = 0;
    if (nd.op == SOUFFLE_OP_MATMUL) {
      ops = 2 * g.nodes[nd.a].shape.back() * O;
    } else if (nd.op == SOUFFLE_OP_REDUCE) {
      const auto& is = g.nodes[nd.in[0]].shape;
      int ax = nd.axis < 0 ? nd.axis + (int)is.size() : nd.axis;
      ops = is[ax] * O;
    } else if (nd.op == SOUFFLE_OP_ELEMENTWISE) {
      ops = O;
    }
    int64_t acc = O;
    for (int j : distinct_inputs(nd)) acc += (nd.op == SOUFFLE_OP_SLICE) ? O : numel(g.nodes[j].shape);
    a.dep[i] = is_mr_op(nd.op) ? 1 : 0;
    a.ops[i] = ops;
    a.acc[i] = acc;
    a.ci[i] = ops >= 3 * acc ? 1 : 0;
    for (int j : distinct_inputs(nd)) a.cons[j].push_back(i);
  }

  // ---- reachability bitsets (descendants), for reuse kinds (§5.1)
  const int W = (n + 63) / 64;
  std::vector<uint64_t> reach((size_t)n * W, 0);
  for (int i = n - 1; i >= 0; --i) {
    uint64_t* ri = &reach[(size_t)i * W];
    for (int c : a.cons[i]) {
      ri[c >> 6] |= 1ull << (c & 63);
      const uint64_t* rc = &reach[(size_t)c * W];
      for (int w = 0; w < W; ++w) ri[w] |= rc[w];
    }
  }
  auto reaches = [&](int x, int y) { return (reach[(size_t)x * W + (y >> 6)] >> (y & 63)) & 1ull; };
  for (int t = 0; t < n; ++t) {
    const auto& cs = a.cons[t];
    if (cs.size() < 2) continue;
    int dep = 0;
    for (size_t x = 0; x < cs.size() && !dep; ++x)
      for (size_t y = x + 1; y < cs.size(); ++y)
        if (reaches(cs[x], cs[y]) || reaches(cs[y], cs[x])) { dep = 1; break; }
    a.reuse_kind[t] = dep;
  }

  // ---- Kahn BFS order over TE->TE edges
  std::vector<std::vector<int>> succ(n);
  std::vector<int> indeg(n, 0);
  for (int i = 0; i < n; ++i) {
    if (g.nodes[i].op == SOUFFLE_OP_PLACEHOLDER) continue;
    for (int j : distinct_inputs(g.nodes[i]))
      if (g.nodes[j].op != SOUFFLE_OP_PLACEHOLDER) { succ[j].push_back(i); indeg[i]++; }
  }
  std::deque<int> q;
  for (int i = 0; i < n; ++i)
    if (g.nodes[i].op != SOUFFLE_OP_PLACEHOLDER && indeg[i] == 0) q.push_back(i);
  while (!q.empty()) {
    int e = q.front();
    q.pop_front();
    a.order.push_back(e);
    auto s = succ[e];
    std::sort(s.begin(), s.end());
    for (int x : s)
      if (--indeg[x] == 0) q.push_back(x);
  }

  // ---- levels
  for (int i = 0; i < n; ++i) {
    if (g.nodes[i].op == SOUFFLE_OP_PLACEHOLDER) continue;
    int lv = 0;
    bool any = false;
    for (int j : node_inputs(g.nodes[i]))
      if (g.nodes[j].op != SOUFFLE_OP_PLACEHOLDER) { lv = std::max(lv, a.level[j] + 1); any = true; }
    a.level[i] = any ? lv : 0;
  }

  // ---- resources and greedy partition (§5.4, Alg. 1 lines 2-9)
  for (int i = 0; i < n; ++i) {
    if (!a.ci[i]) continue;
    const Node& nd = g.nodes[i];
    if (nd.res_override) {
      a.res[i] = Resources{nd.r_grid, nd.r_smem, nd.r_regs, nd.r_threads};
    } else {
      a.res[i] = default_resources(g, i);
    }
  }
  int sp = 0;
  bool have = false;
  Resources cur;
  for (int e : a.order) {
    if (a.ci[e]) {
      const Resources& r = a.res[e];
      if (!have) {
        cur = r;
        have = true;
      } else {
        Resources cand{std::max(cur.grid, r.grid), std::max(cur.smem, r.smem), std::max(cur.regs, r.regs),
                       std::max(cur.threads, r.threads)};
        if (fits(dev, cand)) {
          cur = cand;
        } else {
          ++sp;
          cur = r;
        }
      }
    }
    a.assign[e] = sp;
  }
  a.num_sp = a.order.empty() ? 0 : sp + 1;

  // ---- horizontal groups (§6.1)
  std::vector<int> mm;
  for (int i = 0; i < n; ++i)
    if (g.nodes[i].op == SOUFFLE_OP_MATMUL) mm.push_back(i);
  auto K = [&](int i) { return g.nodes[g.nodes[i].a].shape.back(); };
  for (size_t x = 0; x < mm.size(); ++x) {
    int i = mm[x];
    if (a.hgid[i] >= 0) continue;
    const Node& ni = g.nodes[i];
    std::vector<int> mem;
    for (size_t y = x + 1; y < mm.size(); ++y) {
      int j = mm[y];
      const Node& nj = g.nodes[j];
      if (a.hgid[j] >= 0 || a.assign[j] != a.assign[i] || a.level[j] != a.level[i]) continue;
      if (nj.a != ni.a || nj.trans_b != ni.trans_b || nj.prec != ni.prec || K(j) != K(i)) continue;
      if (g.nodes[nj.b].shape.size() != g.nodes[ni.b].shape.size()) continue;
      mem.push_back(j);
    }
    if (!mem.empty()) {
      int gid = (int)a.hkind.size();
      a.hkind.push_back(0);
      a.hgid[i] = gid;
      for (int j : mem) a.hgid[j] = gid;
    }
  }
  for (size_t x = 0; x < mm.size(); ++x) {
    int i = mm[x];
    if (a.hgid[i] >= 0 || g.nodes[i].shape.size() != 2) continue;
    const Node& ni = g.nodes[i];
    std::vector<int> mem;
    for (size_t y = x + 1; y < mm.size(); ++y) {
      int j = mm[y];
      const Node& nj = g.nodes[j];
      if (a.hgid[j] >= 0 || nj.shape.size() != 2 || a.assign[j] != a.assign[i] || a.level[j] != a.level[i]) continue;
      if (nj.prec != ni.prec || K(j) != K(i) || nj.shape[1] != ni.shape[1]) continue;
      mem.push_back(j);
    }
    if (!mem.empty()) {
      int gid = (int)a.hkind.size();
      a.hkind.push_back(1);
      a.hgid[i] = gid;
      for (int j : mem) a.hgid[j] = gid;
    }
  }
}

// ------------------------------------------------------------------ index maps (§5.2, §6.2)
static void unravel(int64_t f, const std::vector<int64_t>& s, int64_t* idx) {
  for (int d = (int)s.size() - 1; d >= 0; --d) {
    idx[d] = f % s[d];
    f /= s[d];
  }
}
static int64_t ravel(const int64_t* idx, const std::vector<int64_t>& s) {
  int64_t f = 0;
  for (size_t d = 0; d < s.size(); ++d) f = f * s[d] + idx[d];
  return f;
}

void or_map(const Graph& g, int node, int pos, const int64_t* idx, int64_t* out) {
  const Node& n = g.nodes[node];
  const int nd = (int)n.shape.size();
  switch (n.op) {
    case SOUFFLE_OP_ELEMENTWISE: {
      const auto& is = g.nodes[n.in[pos]].shape;
      int off = nd - (int)is.size();
      for (size_t d = 0; d < is.size(); ++d) out[d] = is[d] == 1 ? 0 : idx[d + off];
      break;
    }
    case SOUFFLE_OP_RESHAPE: unravel(ravel(idx, n.shape), g.nodes[n.in[0]].shape, out); break;
    case SOUFFLE_OP_PERMUTE:
      for (int k = 0; k < nd; ++k) out[n.perm[k]] = idx[k];
      break;
    case SOUFFLE_OP_SLICE:
      for (int d = 0; d < nd; ++d) out[d] = n.begin[d] + idx[d] * n.stride[d];
      break;
    case SOUFFLE_OP_ROLL:   // quasi-affine: (i - shift) mod n
      for (int d = 0; d < nd; ++d) {
        const int64_t m = n.shape[d];
        out[d] = ((idx[d] - n.shifts[d]) % m + m) % m;
      }
      break;
    default: throw std::runtime_error("or_map on a non-OR TE");
  }
}

// first OR-only path from t back to s in operand order (depth first)
static bool or_path(const Graph& g, int t, int s, std::vector<std::pair<int, int>>& path) {
  if (t == s) return true;
  const Node& n = g.nodes[t];
  if (!is_or_op(n.op)) return false;
  for (size_t pos = 0; pos < n.in.size(); ++pos) {
    path.push_back({t, (int)pos});
    if (or_path(g, n.in[pos], s, path)) return true;
    path.pop_back();
  }
  return false;
}

bool index_map(const Graph& g, int t, int s, std::vector<int64_t>& out) {
  std::vector<std::pair<int, int>> path;
  if (!or_path(g, t, s, path)) return false;
  const auto& ts = g.nodes[t].shape;
  int64_t N = numel(ts);
  out.resize(N);
  int64_t a[8], b[8];
  for (int64_t f = 0; f < N; ++f) {
    unravel(f, ts, a);
    int64_t* cur = a;
    int64_t* nxt = b;
    for (auto& pr : path) {
      or_map(g, pr.first, pr.second, cur, nxt);
      std::swap(cur, nxt);
    }
    out[f] = ravel(cur, g.nodes[s].shape);
  }
  return true;
}

}  // namespace souffle
