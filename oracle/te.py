"""Oracle: plain fp64 interpreter of an UNFUSED tensor-expression (TE) program.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
--impl reference legs may import this.  It shares no code with the CUDA path.

What a TE is (§3; Fig. 2): a pure function defining every element of
its output over an iteration domain equal to the output shape, with optional reduce axes.  The
fused kernels must reproduce this definition up to floating-point reassociation, because every
Souffle transformation is semantics-preserving (§6).

Per-op semantics (the readings are listed in DESIGN.md "Readings of the paper"):
  matmul(a, b, trans_b, prec):  out[..., m, n] = sum_k A[..., m, k] * B[..., k, n]
        (B = b^T when trans_b).  Batch dims of a and b equal, or b is 2-D and broadcast.
        prec == "bf16": both operands are first rounded to bf16 (RNE) -- "FP16 for GEMM, FP32 for
        everything else" (§7.1, bf16 on B200).  Only applied when
        bf16_operands=True (the `emulate_bf16_operands` mode).
  ew(fn, inputs, scalar): numpy broadcasting over trailing dims.
  reduce(fn, axis, keepdim): sum / max / mean over ONE axis.
  reshape / permute / strided slice: pure index maps (one-relies-on-one, §5.2).
  roll(shifts): cyclic shift, out[..., i, ...] = in[..., (i - shift) mod n, ...] per dim
        (torch.roll / np.roll semantics) -- a quasi-affine (mod) index map (§5.2
        "quasi-affine maps"); Swin-Transformer's shifted windows (Table 2).

Two evaluation modes: vectorised numpy (default) and `brute=True`, which evaluates every output
element by its definition in pure Python loops (tiny shapes only) and pins the vectorised mode.
"""
from __future__ import annotations

import itertools
import math

import numpy as np

UNARY = {"exp", "tanh", "sigmoid", "relu", "gelu_erf", "rsqrt", "neg"}
BINARY = {"add", "sub", "mul", "div", "max"}
SCALAR = {"add_scalar", "mul_scalar"}


# ---------------------------------------------------------------- shape inference
def bcast_shape(*shapes):
    nd = max(len(s) for s in shapes)
    out = []
    for d in range(nd):
        dims = [s[d - (nd - len(s))] for s in shapes if d - (nd - len(s)) >= 0]
        m = max(dims)
        for x in dims:
            if x != 1 and x != m:
                raise ValueError(f"not broadcastable: {shapes}")
        out.append(m)
    return tuple(out)


def slice_len(b, e, s):
    return max(0, -(-(e - b) // s))


def infer_shapes(spec):
    shapes = []
    for n in spec["nodes"]:
        op = n["op"]
        if op == "placeholder":
            shp = tuple(n["shape"])
        elif op == "matmul":
            a, b = shapes[n["a"]], shapes[n["b"]]
            K = a[-1]
            if n["trans_b"]:
                N, Kb = b[-2], b[-1]
            else:
                Kb, N = b[-2], b[-1]
            assert K == Kb, (a, b)
            assert len(b) == 2 or b[:-2] == a[:-2], (a, b)
            shp = tuple(a[:-1]) + (N,)
        elif op == "ew":
            shp = bcast_shape(*[shapes[i] for i in n["in"]])
        elif op == "reduce":
            s = list(shapes[n["in"]])
            ax = n["axis"] % len(s)
            if n["keepdim"]:
                s[ax] = 1
            else:
                s.pop(ax)
            shp = tuple(s)
        elif op == "reshape":
            shp = tuple(n["shape"])
            assert math.prod(shp) == math.prod(shapes[n["in"]])
        elif op == "permute":
            s = shapes[n["in"]]
            shp = tuple(s[p] for p in n["perm"])
        elif op == "slice":
            shp = tuple(slice_len(b, e, st) for b, e, st in zip(n["begin"], n["end"], n["stride"]))
        elif op == "roll":
            shp = tuple(shapes[n["in"]])
            assert len(n["shifts"]) == len(shp)
        else:
            raise ValueError(op)
        shapes.append(shp)
    return shapes


# ---------------------------------------------------------------- bf16 rounding (oracle's own)
def round_bf16(x):
    """Round fp64 values to the nearest bf16 value (8 significant bits), ties to even.
    Independent of synth/ and of the GPU's cvt.rn.bf16x2.f32; finite, normal-range inputs."""
    x = np.asarray(x, dtype=np.float64)
    m, e = np.frexp(x)                  # x = m * 2**e, 0.5 <= |m| < 1
    return np.ldexp(np.round(m * 256.0) / 256.0, e)   # np.round is round-half-even


# ---------------------------------------------------------------- scalar definitions
def _gelu(x):
    return 0.5 * x * (1.0 + math.erf(x / math.sqrt(2.0)))


def unary_scalar(fn, x):
    if fn == "exp":
        return math.exp(x)
    if fn == "tanh":
        return math.tanh(x)
    if fn == "sigmoid":
        return 1.0 / (1.0 + math.exp(-x))
    if fn == "relu":
        return x if x > 0 else 0.0
    if fn == "gelu_erf":
        return _gelu(x)
    if fn == "rsqrt":
        return 1.0 / math.sqrt(x)
    if fn == "neg":
        return -x
    raise ValueError(fn)


def binary_scalar(fn, a, b):
    if fn == "add":
        return a + b
    if fn == "sub":
        return a - b
    if fn == "mul":
        return a * b
    if fn == "div":
        return a / b
    if fn == "max":
        return max(a, b)
    raise ValueError(fn)


def unary_vec(fn, x):
    if fn == "exp":
        return np.exp(x)
    if fn == "tanh":
        return np.tanh(x)
    if fn == "sigmoid":
        return 1.0 / (1.0 + np.exp(-x))
    if fn == "relu":
        return np.maximum(x, 0.0)
    if fn == "gelu_erf":
        from scipy.special import erf
        return 0.5 * x * (1.0 + erf(x / np.sqrt(2.0)))
    if fn == "rsqrt":
        return 1.0 / np.sqrt(x)
    if fn == "neg":
        return -x
    raise ValueError(fn)


def binary_vec(fn, a, b):
    if fn == "add":
        return a + b
    if fn == "sub":
        return a - b
    if fn == "mul":
        return a * b
    if fn == "div":
        return a / b
    if fn == "max":
        return np.maximum(a, b)
    raise ValueError(fn)


# ---------------------------------------------------------------- evaluation
def evaluate(spec, inputs, bf16_operands=False, brute=False):
    """Evaluate every node of `spec` (TEs in id order, §4) in fp64.

    inputs: dict placeholder id -> array (stored values; widened exactly to fp64).
    Returns list of fp64 arrays, one per node (all intermediates kept)."""
    shapes = infer_shapes(spec)
    vals = []
    for i, n in enumerate(spec["nodes"]):
        op = n["op"]
        if op == "placeholder":
            v = np.asarray(inputs[i], dtype=np.float64).reshape(shapes[i])
        elif brute:
            v = _brute(n, vals, shapes, i, bf16_operands)
        else:
            v = _vec(n, vals, bf16_operands)
        assert v.shape == shapes[i], (i, v.shape, shapes[i])
        vals.append(v)
    return vals


def _vec(n, vals, bf16_operands):
    op = n["op"]
    if op == "matmul":
        a, b = vals[n["a"]], vals[n["b"]]
        if bf16_operands and n["prec"] == "bf16":
            a, b = round_bf16(a), round_bf16(b)
        if n["trans_b"]:
            b = np.swapaxes(b, -1, -2)
        return np.matmul(a, b)
    if op == "ew":
        fn = n["fn"]
        xs = [vals[j] for j in n["in"]]
        if fn in UNARY:
            return unary_vec(fn, xs[0])
        if fn in BINARY:
            return binary_vec(fn, xs[0], xs[1])
        if fn == "add_scalar":
            return xs[0] + n["scalar"]
        if fn == "mul_scalar":
            return xs[0] * n["scalar"]
        raise ValueError(fn)
    if op == "reduce":
        x = vals[n["in"]]
        f = {"sum": np.sum, "max": np.max, "mean": np.mean}[n["fn"]]
        return f(x, axis=n["axis"], keepdims=bool(n["keepdim"]))
    if op == "reshape":
        return vals[n["in"]].reshape(tuple(n["shape"]))
    if op == "permute":
        return np.transpose(vals[n["in"]], tuple(n["perm"]))
    if op == "slice":
        sl = tuple(slice(b, e, s) for b, e, s in zip(n["begin"], n["end"], n["stride"]))
        return vals[n["in"]][sl]
    if op == "roll":
        return np.roll(vals[n["in"]], tuple(n["shifts"]), axis=tuple(range(len(n["shifts"]))))
    raise ValueError(op)


def _bidx(idx, in_shape):
    """Broadcast index: output index -> input index (numpy right-aligned broadcasting)."""
    off = len(idx) - len(in_shape)
    return tuple(0 if in_shape[d] == 1 else idx[d + off] for d in range(len(in_shape)))


def _brute(n, vals, shapes, i, bf16_operands):
    """Element-by-element definition, pure Python (§3: each output element individually)."""
    op = n["op"]
    shp = shapes[i]
    out = np.zeros(shp, dtype=np.float64)
    for idx in itertools.product(*[range(d) for d in shp]):
        if op == "matmul":
            A, B = vals[n["a"]], vals[n["b"]]
            bsh = shapes[n["b"]]
            K = shapes[n["a"]][-1]
            bat = idx[:-2]
            m, nn = idx[-2], idx[-1]
            acc = 0.0
            for k in range(K):
                av = float(A[bat + (m, k)])
                bb = bat if len(bsh) > 2 else ()
                bv = float(B[bb + ((nn, k) if n["trans_b"] else (k, nn))])
                if bf16_operands and n["prec"] == "bf16":
                    av, bv = float(round_bf16(av)), float(round_bf16(bv))
                acc += av * bv
            out[idx] = acc
        elif op == "ew":
            fn = n["fn"]
            xs = [float(vals[j][_bidx(idx, shapes[j])]) for j in n["in"]]
            if fn in UNARY:
                out[idx] = unary_scalar(fn, xs[0])
            elif fn in BINARY:
                out[idx] = binary_scalar(fn, xs[0], xs[1])
            elif fn == "add_scalar":
                out[idx] = xs[0] + n["scalar"]
            else:
                out[idx] = xs[0] * n["scalar"]
        elif op == "reduce":
            src = vals[n["in"]]
            ish = shapes[n["in"]]
            ax = n["axis"] % len(ish)
            base = list(idx)
            if not n["keepdim"]:
                base.insert(ax, 0)
            acc = None
            for r in range(ish[ax]):
                base[ax] = r
                x = float(src[tuple(base)])
                if acc is None:
                    acc = x
                elif n["fn"] == "max":
                    acc = max(acc, x)
                else:
                    acc += x
            out[idx] = acc / ish[ax] if n["fn"] == "mean" else acc
        elif op == "reshape":
            flat = 0
            for d, v in zip(shp, idx):
                flat = flat * d + v
            ish = shapes[n["in"]]
            src = []
            for d in reversed(ish):
                src.append(flat % d)
                flat //= d
            out[idx] = vals[n["in"]][tuple(reversed(src))]
        elif op == "permute":
            perm = n["perm"]
            src = [0] * len(perm)
            for k, p in enumerate(perm):
                src[p] = idx[k]
            out[idx] = vals[n["in"]][tuple(src)]
        elif op == "slice":
            src = tuple(b + v * s for b, v, s in zip(n["begin"], idx, n["stride"]))
            out[idx] = vals[n["in"]][src]
        elif op == "roll":
            src = tuple((v - sh) % d for v, sh, d in zip(idx, n["shifts"], shp))
            out[idx] = vals[n["in"]][src]
        else:
            raise ValueError(op)
    return out
