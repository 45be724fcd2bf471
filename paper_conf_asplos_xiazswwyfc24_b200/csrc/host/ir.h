// Internal IR of libsouffle: the TE program (§3) and its analysis results
// (§5).  Host-only C++17.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../../include/souffle.h"

namespace souffle {

struct Node {
  int op = SOUFFLE_OP_PLACEHOLDER;
  std::vector<int64_t> shape;
  int dtype = SOUFFLE_F32;  // storage dtype of placeholders; computed TEs are fp32
  int is_const = 0;
  // matmul
  int a = -1, b = -1, trans_b = 0, prec = SOUFFLE_F32;
  // elementwise
  int fn = -1;
  std::vector<int> in;  // ew inputs; reduce/reshape/permute/slice use in[0]
  double scalar = 0.0;
  // reduce
  int axis = 0, keepdim = 0;
  // permute / slice
  std::vector<int> perm;
  std::vector<int64_t> begin, end, stride;
  // roll
  std::vector<int64_t> shifts;
  // partition resource override (§5.4 "Get required resource")
  bool res_override = false;
  int64_t r_grid = 0, r_smem = 0;
  int r_regs = 0, r_threads = 0;
};

struct Graph {
  std::vector<Node> nodes;
  std::vector<int> outputs;
};

int64_t numel(const std::vector<int64_t>& s);
std::vector<int> node_inputs(const Node& n);          // operand order, duplicates kept
std::vector<int> distinct_inputs(const Node& n);      // sorted unique
bool is_or_op(int op);
bool is_mr_op(int op);

struct Resources {
  int64_t grid = 0, smem = 0;
  int32_t regs = 0, threads = 0;
};

struct Analysis {
  int n = 0;
  std::vector<int> dep;             // 0 OR, 1 MR, -1 placeholder       (§5.2)
  std::vector<int> ci;              // 1 compute-intensive                (§5.3)
  std::vector<int64_t> ops, acc;
  std::vector<std::vector<int>> cons;  // sorted distinct consumer TEs   (§5.1)
  std::vector<int> reuse_kind;      // -1 none, 0 spatial, 1 temporal
  std::vector<int> order;           // Kahn BFS (Alg. 1 line 2)
  std::vector<int> level;           // ASAP level
  std::vector<Resources> res;       // per CI TE
  std::vector<int> assign;          // TE -> subprogram
  int num_sp = 0;
  std::vector<int> hgid;            // horizontal group id (§6.1)
  std::vector<int> hkind;           // per group: 0 N-concat, 1 M-concat
};

void analyse(const Graph& g, const souffle_device_desc& dev, Analysis& a);
bool fits(const souffle_device_desc& dev, const Resources& r);
Resources default_resources(const Graph& g, int te);   // library tile-table policy
// §5.2/§6.2 index map from t back to s by substitution; empty if no OR-only path
bool index_map(const Graph& g, int t, int s, std::vector<int64_t>& out);
// map an output index of OR TE `node` to its input at operand position `pos`
void or_map(const Graph& g, int node, int pos, const int64_t* idx, int64_t* out_idx);

}  // namespace souffle
