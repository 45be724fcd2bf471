"""Oracle: the paper's TE transformations evaluated element by element (TEST INFRASTRUCTURE ONLY).

  hfused_mconcat()  Fig. 3: C = te.compute((M1+M2, N), sum_rk
                    if_then_else(i<M1, A1[i,rk], A2[i-M1,rk]) * if_then_else(i<M1, B1[rk,j], B2[rk,j])).
                    (The printed A2[i, rk] must read A2[i-4, rk]; reading R6.)
  hfused_nconcat()  §6.1: independent TEs sharing the input tensor; outputs concatenated
                    along N, predicate on the output column region, shared input read once.
  vfused_eval()     §6.2: an OR chain evaluated as ONE TE -- every output element is
                    computed from the chain's leaves through the composed index maps.
All three must equal the unfused program (semantics preservation, L1052-1060).
"""
from __future__ import annotations

import itertools

import numpy as np

from .analysis import OR_OPS, or_map
from .te import binary_scalar, infer_shapes, unary_scalar, _bidx


def hfused_mconcat(As, Bs):
    """As[g]: [M_g, K], Bs[g]: [K, N] (trans_b = 0).  Returns the fused [sum M_g, N] tensor."""
    Ms = [a.shape[0] for a in As]
    K, N = As[0].shape[1], Bs[0].shape[1]
    out = np.zeros((sum(Ms), N))
    for i in range(sum(Ms)):
        g, base = 0, 0
        while i >= base + Ms[g]:          # predicate chain of if_then_else on the output region
            base += Ms[g]
            g += 1
        for j in range(N):
            out[i, j] = sum(float(As[g][i - base, rk]) * float(Bs[g][rk, j]) for rk in range(K))
    return out


def hfused_nconcat(A, Bs, trans_b=1):
    """A: [M, K] shared; Bs[g]: [N_g, K] (trans_b=1) -> fused [M, sum N_g]."""
    Ns = [b.shape[0] if trans_b else b.shape[1] for b in Bs]
    M, K = A.shape
    out = np.zeros((M, sum(Ns)))
    for j in range(sum(Ns)):
        g, base = 0, 0
        while j >= base + Ns[g]:
            base += Ns[g]
            g += 1
        jj = j - base
        for i in range(M):
            out[i, j] = sum(float(A[i, rk]) * float(Bs[g][jj, rk] if trans_b else Bs[g][rk, jj]) for rk in range(K))
    return out


def vfused_eval(spec, vals, t, leaves):
    """Evaluate TE t as one vertically-transformed TE: recursion through OR TEs down to `leaves`
    (tensors treated as inputs of the fused TE), composing index maps on the way."""
    shapes = infer_shapes(spec)
    nodes = spec["nodes"]

    def value(node, idx):
        if node in leaves or nodes[node]["op"] not in OR_OPS:
            return float(vals[node][tuple(idx)])
        n = nodes[node]
        if n["op"] == "ew":
            xs = [value(j, or_map(n, shapes, node, pos, idx)) for pos, j in enumerate(n["in"])]
            fn = n["fn"]
            if len(xs) == 2:
                return binary_scalar(fn, xs[0], xs[1])
            if fn == "add_scalar":
                return xs[0] + n["scalar"]
            if fn == "mul_scalar":
                return xs[0] * n["scalar"]
            return unary_scalar(fn, xs[0])
        return value(n["in"], or_map(n, shapes, node, 0, idx))

    out = np.zeros(shapes[t])
    for idx in itertools.product(*[range(d) for d in shapes[t]]):
        out[idx] = value(t, list(idx))
    return out
