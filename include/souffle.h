/* souffle.h — C ABI of libsouffle: build a tensor-expression (TE) program, partition it into
 * subprograms with Souffle's dataflow-and-resource analysis, and execute every subprogram as ONE
 * persistent sm_100a kernel.
 *
 * Paper: Xia et al., "Optimizing Deep Learning Inference via Global Analysis and Tensor
 * Expressions", ASPLOS'24 (text at /root/reference/PAPER.md, cited below as P:L<line>).
 *
 *   TE program input ............ §3, §4 P:L607-610 (Fig. 2)
 *   global analysis ............. §5.1-5.3
 *   resource-aware partition .... §5.4, Algorithm 1 lines 2-9 P:L1257-1269
 *   TE transformations .......... §6.1-6.2 P:L1062-1153 (horizontal / vertical)
 *   one kernel per subprogram ... §4, §6.4 P:L1169-1176 (global sync between stages)
 *
 * Conventions (all entry points):
 *   - Every call returns souffle_status; 0 == SOUFFLE_OK.  On error a thread-local message is
 *     available from souffle_last_error() until the next souffle_* call on the same thread.
 *   - Handles (souffle_graph, souffle_plan) are created and destroyed only by the library.
 *     Destroying NULL is a no-op.  A plan is independent of its graph after creation.
 *   - Tensors are dense int32 ids in creation order; creation order is a topological order.
 *   - Shapes are int64 arrays, row-major (last dim contiguous), ndim 1..8.
 *   - Graph building, analysis, partitioning and plan introspection are pure host code and work
 *     on a machine without a GPU.  Execution needs an sm_100 device: there is NO CPU fallback
 *     (SOUFFLE_E_UNSUPPORTED otherwise).
 *   - Device memory is owned by the caller (PyTorch in the Python binding).  Pointers passed to
 *     souffle_bind / souffle_run are borrowed and must stay valid until the stream work ends.
 *   - Streams are passed as `void*` (a cudaStream_t; NULL = legacy default stream).
 */
#ifndef SOUFFLE_H_
#define SOUFFLE_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t souffle_status;
enum {
  SOUFFLE_OK = 0,
  SOUFFLE_E_INVALID_ARG = 1, /* bad handle / id / pointer / enum value                          */
  SOUFFLE_E_SHAPE = 2,       /* shapes do not conform to the op's definition                     */
  SOUFFLE_E_UNSUPPORTED = 3, /* op/dtype combination not implemented, or no sm_100 device         */
  SOUFFLE_E_RESOURCE = 4,    /* a cooperative launch cannot be co-resident on the device          */
  SOUFFLE_E_CUDA = 5,        /* a CUDA runtime/driver call failed (message has the CUDA string)   */
  SOUFFLE_E_STATE = 6,       /* wrong call order, e.g. souffle_run before every input is bound    */
  SOUFFLE_E_OOM = 7          /* host allocation failed                                            */
};

const char* souffle_last_error(void);
const char* souffle_version(void);

typedef struct souffle_graph_s* souffle_graph;
typedef struct souffle_plan_s* souffle_plan;
typedef int32_t souffle_tensor;

/* storage dtypes of placeholders; every computed TE is fp32 by definition */
enum { SOUFFLE_F32 = 0, SOUFFLE_BF16 = 1 };

/* node kinds reported by souffle_graph_node */
enum { SOUFFLE_OP_PLACEHOLDER = 0, SOUFFLE_OP_MATMUL = 1, SOUFFLE_OP_ELEMENTWISE = 2,
       SOUFFLE_OP_REDUCE = 3, SOUFFLE_OP_RESHAPE = 4, SOUFFLE_OP_PERMUTE = 5, SOUFFLE_OP_SLICE = 6,
       SOUFFLE_OP_ROLL = 7 };

/* elementwise functions (one-relies-on-one TEs, §5.2).  Binary ops use numpy
 * broadcasting over trailing dims; *_SCALAR ops take the `scalar` argument. */
enum {
  SOUFFLE_EW_ADD = 0, SOUFFLE_EW_SUB = 1, SOUFFLE_EW_MUL = 2, SOUFFLE_EW_DIV = 3, SOUFFLE_EW_MAX = 4,
  SOUFFLE_EW_EXP = 5, SOUFFLE_EW_TANH = 6, SOUFFLE_EW_SIGMOID = 7, SOUFFLE_EW_RELU = 8,
  SOUFFLE_EW_GELU_ERF = 9, SOUFFLE_EW_RSQRT = 10, SOUFFLE_EW_NEG = 11,
  SOUFFLE_EW_ADD_SCALAR = 12, SOUFFLE_EW_MUL_SCALAR = 13
};
/* reductions (one-relies-on-many TEs with one reduce axis, §5.2) */
enum { SOUFFLE_RED_SUM = 0, SOUFFLE_RED_MAX = 1, SOUFFLE_RED_MEAN = 2 };

/* ------------------------------------------------------------------ graph building (§3, §4) */
souffle_status souffle_graph_create(souffle_graph* out);
souffle_status souffle_graph_destroy(souffle_graph g);

/* A graph input.  dtype: storage dtype (SOUFFLE_F32 / SOUFFLE_BF16).  is_constant marks weights
 * (used for reuse/temporal analysis and for the weight-prefetch plan; values still come from
 * souffle_bind). */
souffle_status souffle_placeholder(souffle_graph g, int32_t ndim, const int64_t* shape, int32_t dtype,
                                   int32_t is_constant, souffle_tensor* out);

/* out[..., m, n] = sum_k A[..., m, k] * B[..., k, n], B = b^T if trans_b (b stored [.., N, K]).
 * a: [..., M, K]; b: [..., K, N] or [..., N, K]; b's batch dims equal a's, or b is 2-D.
 * precision SOUFFLE_BF16: both operands are rounded to bf16 (RNE) first, fp32 accumulation
 * ("FP16 for GEMM, FP32 for everything else"; bf16 on B200).
 * precision SOUFFLE_F32: fp32 operands (a bf16-stored operand is used exactly), fp32 FMA. */
souffle_status souffle_matmul(souffle_graph g, souffle_tensor a, souffle_tensor b, int32_t trans_b,
                              int32_t precision, souffle_tensor* out);
souffle_status souffle_elementwise(souffle_graph g, int32_t op, int32_t n_in, const souffle_tensor* in,
                                   double scalar, souffle_tensor* out);
souffle_status souffle_reduce(souffle_graph g, int32_t op, souffle_tensor in, int32_t axis, int32_t keepdim,
                              souffle_tensor* out);
souffle_status souffle_reshape(souffle_graph g, souffle_tensor in, int32_t ndim, const int64_t* shape,
                               souffle_tensor* out);
/* out.shape[i] = in.shape[perm[i]]  (numpy transpose) */
souffle_status souffle_permute(souffle_graph g, souffle_tensor in, const int32_t* perm, souffle_tensor* out);
/* strided slice, half-open [begin, end) with positive stride per dim (Fig. 4) */
souffle_status souffle_slice(souffle_graph g, souffle_tensor in, const int64_t* begin, const int64_t* end,
                             const int64_t* stride, souffle_tensor* out);
/* cyclic shift (torch.roll / np.roll): out[.., i_d, ..] = in[.., (i_d - shifts[d]) mod n_d, ..] for every
 * dim d (shifts has ndim entries, any sign).  A one-relies-on-one TE whose index map is quasi-affine
 * (mod by a constant, §5.2 P:L897-898 "quasi-affine maps"): Swin-Transformer's shifted windows
 * (Table 2).  Errors: E_INVALID_ARG on a null argument. */
souffle_status souffle_roll(souffle_graph g, souffle_tensor in, const int64_t* shifts, souffle_tensor* out);
souffle_status souffle_mark_output(souffle_graph g, souffle_tensor t);

/* graph introspection (used by tests to compare with the oracle's own builders) */
souffle_status souffle_graph_num_nodes(souffle_graph g, int32_t* n);
souffle_status souffle_graph_node(souffle_graph g, souffle_tensor t, int32_t* op, int32_t* ndim,
                                  int64_t* shape /* >= 8 entries */, int32_t* dtype);

/* Override the per-TE resource vector used by the partitioner (§5.4 "Get required resource",
 * P:L994-997).  By default the library derives it from its kernel tile table; the override lets
 * tests feed the paper's Fig. 2 numbers (16/16/64 blocks, 1 KB).  Only CI TEs are consulted. */
souffle_status souffle_set_te_resources(souffle_graph g, souffle_tensor te, int64_t grid, int64_t smem,
                                        int32_t regs, int32_t threads);

/* ------------------------------------------------------------------ device description */
typedef struct {
  int32_t num_sms;
  int64_t smem_per_sm, smem_per_block_max, smem_reserved_per_block;
  int32_t regs_per_sm, max_threads_per_sm, max_blocks_per_sm;
  int32_t rule;       /* 0 = exact per-SM occupancy (default), 1 = paper rule max_grid*max_smem <= C */
  int64_t capacity_C; /* bytes; used only by rule 1 */
} souffle_device_desc;

/* Fills the description of the CUDA device (needs a GPU). */
souffle_status souffle_device_query(int32_t cuda_device, souffle_device_desc* out);
/* Fills the B200 defaults (148 SMs, 228 KB smem/SM, 64K regs) without touching a GPU. */
souffle_status souffle_device_b200(souffle_device_desc* out);

/* ------------------------------------------------------------------ partition (§5.4, Alg. 1) */
/* flags: ablation switches (Table 4: V0..V4) */
enum {
  SOUFFLE_FLAG_UNFUSED = 1u,        /* V0: every TE is its own kernel launch                       */
  SOUFFLE_FLAG_NO_HORIZONTAL = 2u,  /* disable §6.1 horizontal transformation                      */
  SOUFFLE_FLAG_NO_VERTICAL = 4u,    /* disable §6.2 vertical transformation (materialise OR TEs)   */
  SOUFFLE_FLAG_NO_GLOBAL_SYNC = 8u, /* one launch per stage instead of grid barriers (§6.4)        */
  SOUFFLE_FLAG_NO_PREFETCH = 16u,   /* disable cross-stage weight prefetch (§6.5)                  */
  SOUFFLE_FLAG_NO_LN_REWRITE = 32u, /* keep LayerNorm as two dependent reductions                  */
  SOUFFLE_FLAG_NO_PATTERN = 64u     /* generic lowering even where a model pattern kernel matches  */
};
/* Analyses the graph, partitions it and lowers every subprogram to a stage list.  Pure host
 * code.  `dev` may come from souffle_device_query or souffle_device_b200. */
souffle_status souffle_partition(souffle_graph g, const souffle_device_desc* dev, uint32_t flags,
                                 souffle_plan* out);
souffle_status souffle_plan_destroy(souffle_plan p);

/* ------------------------------------------------------------------ plan introspection
 * (what the oracle checks bit-exactly).  Arrays are caller-allocated. */
souffle_status souffle_plan_num_nodes(souffle_plan p, int32_t* n);  /* nodes incl. placeholders */
souffle_status souffle_plan_num_tes(souffle_plan p, int32_t* n);    /* computed nodes only */
souffle_status souffle_plan_num_subprograms(souffle_plan p, int32_t* n);
/* te_to_sp[num_nodes]: subprogram of every node, -1 for placeholders */
souffle_status souffle_plan_assignment(souffle_plan p, int32_t* te_to_sp);
/* order[num_tes]: Kahn-BFS order (Alg. 1 line 2) */
souffle_status souffle_plan_bfs_order(souffle_plan p, int32_t* order);
/* dep_kind: 0 one-relies-on-one (OR), 1 one-relies-on-many (MR), -1 placeholder (§5.2);
 * intensity: 0 memory-, 1 compute-intensive (ratio ops/accesses >= 3, §5.3);
 * grid/smem/regs/threads: the resource vector the partitioner used. Any out pointer may be NULL. */
souffle_status souffle_plan_te_info(souffle_plan p, souffle_tensor te, int32_t* dep_kind, int32_t* intensity,
                                    int64_t* ops, int64_t* accesses, int64_t* grid, int64_t* smem,
                                    int32_t* regs, int32_t* threads);
/* §5.1 reuse: the sorted consumer TEs of tensor t (n = count, <= cap written); kind 0 spatial,
 * 1 temporal, -1 if t is read by fewer than 2 TEs. */
souffle_status souffle_plan_reuse_set(souffle_plan p, souffle_tensor t, int32_t* consumers, int32_t cap,
                                      int32_t* n, int32_t* kind);
/* §5.2/§6.2 composed one-relies-on-one index map from fused_out back to source, enumerated as the
 * flat source offset of every element of fused_out (row-major).  SOUFFLE_E_INVALID_ARG if no
 * path of OR TEs connects them.  src_offset must hold numel(fused_out) entries. */
souffle_status souffle_plan_index_map(souffle_plan p, souffle_tensor fused_out, souffle_tensor source,
                                      int64_t* src_offset);
/* ASAP level and horizontal group (§6.1) of a TE: group -1 if not grouped; kind 0 = concat along
 * N (shared A operand), 1 = concat along M (Fig. 3). */
souffle_status souffle_plan_hgroup(souffle_plan p, souffle_tensor te, int32_t* level, int32_t* group,
                                   int32_t* kind);
/* execution structure: kernel launches per souffle_run, total stages, grid barriers */
souffle_status souffle_plan_exec_info(souffle_plan p, int32_t* launches, int32_t* stages, int32_t* barriers);
/* human-readable dump of the lowered stage list (static buffer, valid until plan destroy) */
souffle_status souffle_plan_describe(souffle_plan p, const char** text);

/* ------------------------------------------------------------------ execution */
/* Bytes of device workspace souffle_run needs (intermediates, barrier words, statistics). */
souffle_status souffle_plan_workspace_bytes(souffle_plan p, size_t* bytes);
/* Bind a device pointer to a placeholder (input/weight) or to a marked output.  Placeholders are
 * read in their declared dtype; outputs are written as fp32, row-major. */
souffle_status souffle_bind(souffle_plan p, souffle_tensor t, void* device_ptr);
/* Zero the workspace once after allocating it (enqueued on `stream`).  souffle_run keeps it in a
 * reusable state afterwards (barrier counters are reset by the last CTA to leave). */
souffle_status souffle_workspace_init(souffle_plan p, void* workspace, void* stream);
/* Enqueue the whole program on `stream`: one cooperative launch per subprogram (or one launch
 * per TE under SOUFFLE_FLAG_UNFUSED).  Asynchronous; never allocates or synchronises.  A plan is
 * tied to the ONE workspace last passed to souffle_workspace_init (E_STATE for any other): to run
 * a model concurrently on several streams, create one plan (and workspace) per stream. */
souffle_status souffle_run(souffle_plan p, void* workspace, void* stream);

/* ------------------------------------------------------------------ debug profiling
 * When enabled, CTA 0 of every launch records %globaltimer at each stage start (after its grid
 * barrier) and the last CTA records the launch end, in the workspace control region.
 * souffle_plan_read_profile synchronises the device and returns one duration (microseconds) per
 * stage in execution order: time from the stage's start to the next stage's start (so it
 * includes the grid barrier that follows the stage).  Debug use only (it synchronises).
 * Changing the flag changes the workspace layout: call it BEFORE souffle_plan_workspace_bytes /
 * souffle_workspace_init (otherwise souffle_run returns E_STATE until they are called again). */
souffle_status souffle_plan_set_profiling(souffle_plan p, int32_t on);
souffle_status souffle_plan_read_profile(souffle_plan p, void* workspace, double* stage_us, int32_t cap,
                                         int32_t* n);
/* Raw %globaltimer stamps (ns): [stages + 1] stage starts / launch end, then 8 sub-stage marks
 * per stage (stage-kind specific, 0 if unused).  cap >= 9 * stages + 1. */
souffle_status souffle_plan_read_profile_raw(souffle_plan p, void* workspace, uint64_t* stamps, int32_t cap,
                                             int32_t* n);

/* Test introspection of the BERT pattern kernel (kernels/bert.cu, host/bert.cpp): byte offset from
 * the workspace base and size of one of its named activation buffers -- "xb" / "l1b" (bf16 [S][H]
 * GEMM A operands), "l1f" / "xf" (fp32 [S][H] residual stream), "qk" (bf16 Q then K, head-major
 * [2*heads][S][64]), "vt" (bf16 V^T [heads][64][S]), "h" (bf16 GELU output [S][F]), "part_o" /
 * "part_2" (fp32 split-K partials [nsplit][S][H]).  Used with SOUFFLE_BERT_STAGES=b,e (run only
 * stages [b, e)) by the stage-isolation tests.  Errors: E_INVALID_ARG (unknown name, NULL
 * pointers), E_UNSUPPORTED (the plan does not use the BERT pattern kernel).  A Swin pattern plan
 * has one region, "trace": one uint64 %globaltimer stamp per launch (CTA 0, after its dependency
 * wait) when the workspace was initialised with SOUFFLE_SWIN_TRACE set. */
souffle_status souffle_plan_debug_region(souffle_plan p, const char* name, int64_t* offset, int64_t* bytes);

#ifdef __cplusplus
}
#endif
#endif /* SOUFFLE_H_ */
