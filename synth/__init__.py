"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no TE semantics, no analysis, no partitioning).
It only draws random numbers from documented seeds and rounds them ONCE to their storage dtype,
so that both sides of every parity check consume bit-identical stored values
(SURVEY.md §8(c) item 9, §8(d) "Synthetic inputs").

Generator: numpy.random.Generator(PCG64(seed)) in fp64, then fp64 -> fp32 (numpy RNE) and, for bf16
storage, fp32 -> bf16 by round-to-nearest-even on the bit pattern.  Seeds: inputs = 1234,
weights = 1000 * layer + slot (slot numbers below).

Workload recipes:
  * BERT (Table 2, §7.1): X ~ N(0,1) fp32 is the post-embedding hidden
    state; GEMM weights W ~ N(0, 1/K) stored [N, K]; biases N(0, 0.02^2); LN gamma = 1 + N(0, 0.1^2),
    beta = N(0, 0.1^2).
  * LSTM (Table 2): x ~ N(0,1) [T, 256]; W_ih, W_hh, b_ih, b_hh ~ U(+-1/sqrt(H)) (PyTorch
    default init, contractive; SURVEY §8(c) tolerances).
  * MMoE (Table 2, reading in DESIGN.md): x ~ N(0,1) [1, 100]; every weight ~ N(0, 1/K),
    biases N(0, 0.02^2).
"""
from __future__ import annotations

import numpy as np

INPUT_SEED = 1234

# ---------------------------------------------------------------- configs (BASELINE.json configs)
BERT_TINY = dict(name="bert_tiny", seq=32, hidden=64, heads=2, ffn=256, layers=1, gemm_dtype="f32",
                 eps=1e-12)
BERT_BASE = dict(name="bert_base", seq=128, hidden=768, heads=12, ffn=3072, layers=12, gemm_dtype="bf16",
                 eps=1e-12)
LSTM_CFG = dict(name="lstm", steps=100, hidden=256, input=256, layers=10, w_dtype="bf16")
MMOE_CFG = dict(name="mmoe", d_in=100, experts=8, expert_dim=16, tasks=2, tower_hidden=8, batch=1,
                w_dtype="f32")

# weight slot numbers inside one BERT layer (seed = 1000*layer + slot)
BERT_SLOTS = dict(Wq=1, bq=2, Wk=3, bk=4, Wv=5, bv=6, Wo=7, bo=8, g1=9, be1=10, W1=11, c1=12, W2=13, c2=14,
                  g2=15, be2=16)


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


# ---------------------------------------------------------------- storage rounding (bit level)
def f32_to_bf16_bits(x) -> np.ndarray:
    """fp32 -> bf16 bit pattern (uint16), round-to-nearest-even on the bits (finite inputs)."""
    u = np.ascontiguousarray(np.asarray(x, dtype=np.float32)).view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) >> 16
    return u.astype(np.uint16)


def bf16_bits_to_f32(b) -> np.ndarray:
    b = np.asarray(b, dtype=np.uint16).astype(np.uint32) << 16
    return b.view(np.float32)


def to_storage(x, dtype: str) -> np.ndarray:
    """Round fp64 draws once to the storage dtype; returns float32 values exactly representable
    in `dtype` ('f32' or 'bf16')."""
    x32 = np.asarray(x, dtype=np.float64).astype(np.float32)
    if dtype == "f32":
        return x32
    if dtype == "bf16":
        return bf16_bits_to_f32(f32_to_bf16_bits(x32))
    raise ValueError(dtype)


def normal(seed, shape, std=1.0, mean=0.0, dtype="f32"):
    return to_storage(mean + std * rng(seed).standard_normal(shape), dtype)


def uniform(seed, shape, bound, dtype="f32"):
    return to_storage(rng(seed).uniform(-bound, bound, size=shape), dtype)


def small_ints(seed, shape, lo=-2, hi=2, dtype="f32"):
    """Integer-valued draws in [lo, hi]: exact in bf16 and fp32, so GEMMs over them are exact."""
    return to_storage(rng(seed).integers(lo, hi + 1, size=shape).astype(np.float64), dtype)


# ---------------------------------------------------------------- BERT
def bert_layer_weights(cfg: dict, layer: int, integer: bool = False) -> dict:
    H, F = cfg["hidden"], cfg["ffn"]
    wd = cfg["gemm_dtype"]
    s = lambda k: 1000 * layer + BERT_SLOTS[k]
    if integer:
        w = lambda k, shp: small_ints(s(k), shp, dtype=wd)
        v = lambda k, shp: small_ints(s(k), shp, dtype="f32")
        g = lambda k, shp: small_ints(s(k), shp, 0, 2, dtype="f32")
    else:
        w = lambda k, shp: normal(s(k), shp, std=1.0 / np.sqrt(shp[1]), dtype=wd)
        v = lambda k, shp: normal(s(k), shp, std=0.02)
        g = lambda k, shp: normal(s(k), shp, std=0.1, mean=1.0)
    p = dict(Wq=w("Wq", (H, H)), bq=v("bq", (H,)), Wk=w("Wk", (H, H)), bk=v("bk", (H,)),
             Wv=w("Wv", (H, H)), bv=v("bv", (H,)), Wo=w("Wo", (H, H)), bo=v("bo", (H,)),
             g1=g("g1", (H,)), W1=w("W1", (F, H)), c1=v("c1", (F,)), W2=w("W2", (H, F)), c2=v("c2", (H,)),
             g2=g("g2", (H,)))
    if integer:
        p["be1"] = small_ints(s("be1"), (H,))
        p["be2"] = small_ints(s("be2"), (H,))
    else:
        p["be1"] = normal(s("be1"), (H,), std=0.1)
        p["be2"] = normal(s("be2"), (H,), std=0.1)
    return p


def bert_input(cfg: dict, seed: int = INPUT_SEED, batch: int = 1) -> np.ndarray:
    shape = (cfg["seq"], cfg["hidden"]) if batch == 1 else (batch, cfg["seq"], cfg["hidden"])
    return normal(seed, shape)


def bert_weights(cfg: dict, integer: bool = False) -> list:
    return [bert_layer_weights(cfg, l, integer) for l in range(cfg["layers"])]


# ---------------------------------------------------------------- LSTM
def lstm_params(cfg: dict, w_dtype: str | None = None) -> list:
    H, I = cfg["hidden"], cfg["input"]
    wd = w_dtype or cfg["w_dtype"]
    b = 1.0 / np.sqrt(H)
    out = []
    for n in range(cfg["layers"]):
        out.append(dict(W=uniform(1000 * n + 1, (4 * H, I if n == 0 else H), b, wd),
                        U=uniform(1000 * n + 2, (4 * H, H), b, wd),
                        b_ih=uniform(1000 * n + 3, (4 * H,), b),
                        b_hh=uniform(1000 * n + 4, (4 * H,), b)))
    return out


def lstm_input(cfg: dict, seed: int = INPUT_SEED) -> np.ndarray:
    return normal(seed, (cfg["steps"], cfg["input"]))


# ---------------------------------------------------------------- MMoE
def mmoe_params(cfg: dict) -> dict:
    D, E, De, T, Th = cfg["d_in"], cfg["experts"], cfg["expert_dim"], cfg["tasks"], cfg["tower_hidden"]
    wd = cfg["w_dtype"]
    p = {}
    for e in range(E):
        p[f"We{e}"] = normal(100 + e, (De, D), std=1 / np.sqrt(D), dtype=wd)
        p[f"be{e}"] = normal(200 + e, (De,), std=0.02)
    for k in range(T):
        p[f"Wg{k}"] = normal(300 + k, (E, D), std=1 / np.sqrt(D), dtype=wd)
        p[f"bg{k}"] = normal(400 + k, (E,), std=0.02)
        p[f"Wt{k}"] = normal(500 + k, (Th, De), std=1 / np.sqrt(De), dtype=wd)
        p[f"bt{k}"] = normal(600 + k, (Th,), std=0.02)
        p[f"Wo{k}"] = normal(700 + k, (1, Th), std=1 / np.sqrt(Th), dtype=wd)
        p[f"bo{k}"] = normal(800 + k, (1,), std=0.02)
    return p


def mmoe_input(cfg: dict, seed: int = INPUT_SEED) -> np.ndarray:
    return normal(seed, (cfg["batch"], cfg["d_in"]))


# ---------------------------------------------------------------- random TE-program specs
# Spec format (a plain data format consumed by oracle/te.py and by the binding's spec builder):
#   {"nodes": [node, ...], "outputs": [ids]}, node ids = list positions (creation order = topological)
#   placeholder: {"op":"placeholder","shape":[..],"dtype":"f32"|"bf16","const":0|1}
#   matmul:      {"op":"matmul","a":i,"b":j,"trans_b":0|1,"prec":"f32"|"bf16"}
#   ew:          {"op":"ew","fn":name,"in":[ids],"scalar":x}
#   reduce:      {"op":"reduce","fn":"sum"|"max"|"mean","in":i,"axis":k,"keepdim":0|1}
#   reshape:     {"op":"reshape","in":i,"shape":[..]}
#   permute:     {"op":"permute","in":i,"perm":[..]}
#   slice:       {"op":"slice","in":i,"begin":[..],"end":[..],"stride":[..]}
UNARY = ["exp", "tanh", "sigmoid", "relu", "gelu_erf", "rsqrt", "neg"]
BINARY = ["add", "sub", "mul", "div", "max"]
SCALAR = ["add_scalar", "mul_scalar"]


def random_spec(seed: int, n_ops: int = 12, dim_choices=(2, 3, 4, 5)) -> dict:
    """Random 2-D TE program over small shapes (structure only; shapes kept consistent here so the
    builder never has to reject).  Used for analysis property tests and generic-executor parity."""
    r = rng(seed)
    nodes, shapes = [], []

    def add(node, shape):
        nodes.append(node)
        shapes.append(tuple(shape))
        return len(nodes) - 1

    M, K = int(r.choice(dim_choices)), int(r.choice(dim_choices))
    x = add(dict(op="placeholder", shape=[M, K], dtype="f32", const=0), (M, K))
    live = [x]
    for _ in range(n_ops):
        kind = r.choice(["mm", "un", "bin", "red", "perm", "scal"])
        src = int(r.choice(live))
        shp = shapes[src]
        if len(shp) != 2:
            continue
        if kind == "mm":
            N = int(r.choice(dim_choices))
            w = add(dict(op="placeholder", shape=[N, shp[1]], dtype="f32", const=1), (N, shp[1]))
            nid = add(dict(op="matmul", a=src, b=w, trans_b=1, prec="f32"), (shp[0], N))
        elif kind == "un":
            fn = str(r.choice(["tanh", "sigmoid", "relu", "neg", "exp"]))
            nid = add(dict(op="ew", fn=fn, **{"in": [src]}, scalar=0.0), shp)
        elif kind == "scal":
            fn = str(r.choice(SCALAR))
            nid = add(dict(op="ew", fn=fn, **{"in": [src]}, scalar=float(r.choice([0.5, -1.0, 2.0]))), shp)
        elif kind == "bin":
            same = [i for i in live if shapes[i] == shp and i != src]
            if same:
                other = int(r.choice(same))
            else:
                other = add(dict(op="placeholder", shape=[shp[1]], dtype="f32", const=1), (shp[1],))
            fn = str(r.choice(["add", "sub", "mul", "max"]))
            nid = add(dict(op="ew", fn=fn, **{"in": [src, other]}, scalar=0.0), shp)
        elif kind == "red":
            fn = str(r.choice(["sum", "max", "mean"]))
            nid = add(dict(op="reduce", fn=fn, **{"in": src}, axis=1, keepdim=1), (shp[0], 1))
        else:
            nid = add(dict(op="permute", **{"in": src}, perm=[1, 0]), (shp[1], shp[0]))
        live.append(nid)
    return {"nodes": nodes, "outputs": [len(nodes) - 1]}


def random_rowwise_spec(seed: int, n_ops: int = 14) -> dict:
    """Random row-wise TE program over one [R, C] domain (structure only): chains of row reductions
    (sum / max / mean, keepdim) and elementwise ops that combine [R, C] tensors with the [R, 1]
    statistics -- the LayerNorm / softmax shape of dependence that the generic executor runs as
    reduction and elementwise stages over the same rows (tensor reuse, §6.5).  R spans several row
    blocks per CTA; C includes ragged widths (not a multiple of 8)."""
    r = rng(seed)
    nodes = []

    def add(node):
        nodes.append(node)
        return len(nodes) - 1

    R = int(r.choice([200, 300, 1000, 4000]))
    C = int(r.choice([8, 24, 49, 64, 130]))
    full = [add(dict(op="placeholder", shape=[R, C], dtype="f32", const=0)) for _ in range(int(r.choice([1, 2, 3])))]
    stats = []
    for _ in range(n_ops):
        kind = r.choice(["red", "red", "bin_stat", "bin_stat", "bin", "un"])
        src = int(r.choice(full))
        if kind == "red":
            fn = str(r.choice(["sum", "max", "mean"]))
            stats.append(add(dict(op="reduce", fn=fn, **{"in": src}, axis=1, keepdim=1)))
        elif kind == "bin_stat" and stats:
            fn = str(r.choice(["sub", "mul", "add"]))
            full.append(add(dict(op="ew", fn=fn, **{"in": [src, int(r.choice(stats))]}, scalar=0.0)))
        elif kind == "bin" and len(full) > 1:
            other = int(r.choice([i for i in full if i != src]))
            full.append(add(dict(op="ew", fn=str(r.choice(["add", "mul", "max"])), **{"in": [src, other]}, scalar=0.0)))
        else:
            full.append(add(dict(op="ew", fn=str(r.choice(["tanh", "sigmoid", "neg"])), **{"in": [src]}, scalar=0.0)))
    outs = [full[-1]] + ([stats[-1]] if stats else [])
    return {"nodes": nodes, "outputs": outs}


def spec_inputs(spec: dict, seed: int, integer: bool = False) -> dict:
    """Seeded values for every placeholder of a spec (dict id -> float32 array in storage dtype)."""
    out = {}
    for i, n in enumerate(spec["nodes"]):
        if n["op"] != "placeholder":
            continue
        if integer:
            out[i] = small_ints(seed * 7919 + i, tuple(n["shape"]), dtype=n["dtype"])
        else:
            out[i] = normal(seed * 7919 + i, tuple(n["shape"]), std=0.5, dtype=n["dtype"])
    return out


# ---------------------------------------------------------------- EfficientNet sub-modules M0-M9
# PAPER.md Fig. 5 / Fig. 6 (L1511-1564): the squeeze-and-excitation sub-module of EfficientNet-b0's
# MBConv blocks "repeats many times with different input sizes (M0 to M9)".  The 10 distinct
# (expanded channels C, feature map H x H, squeeze channels S) of efficientnet_b0's 16 blocks
# (torchvision: S = max(1, block input channels // 4)), in network order (reading R20).
SE_CONFIGS = [
    dict(name=f"M{i}", hw=h, channels=c, squeeze=s)
    for i, (c, h, s) in enumerate([(32, 112, 8), (96, 56, 4), (144, 56, 6), (144, 28, 6), (240, 28, 10),
                                   (240, 14, 10), (480, 14, 20), (672, 14, 28), (672, 7, 28), (1152, 7, 48)])
]


def se_input(cfg: dict, seed: int = INPUT_SEED) -> np.ndarray:
    """x [H*W, C] fp32 ~ N(0, 1): the depthwise-conv output the sub-module rescales (NHWC, batch 1)."""
    return normal(seed, (cfg["hw"] * cfg["hw"], cfg["channels"]))


def se_params(cfg: dict) -> dict:
    """fc1 [S, C] ~ N(0, 1/C), b1 N(0, 0.02^2); fc2 [C, S] ~ N(0, 1/S), b2 N(0, 0.02^2); fp32."""
    C, S = cfg["channels"], cfg["squeeze"]
    return dict(W1=normal(701, (S, C), std=1.0 / np.sqrt(C)), b1=normal(702, (S,), std=0.02),
                W2=normal(703, (C, S), std=1.0 / np.sqrt(S)), b2=normal(704, (C,), std=0.02))


# ---------------------------------------------------------------- EfficientNet MBConv blocks M0-M9
# The first efficientnet_b0 block (torchvision MBConvConfig) with each sub-module shape of SE_CONFIGS:
# (input channels, output channels, expand ratio, depthwise kernel, stride, input height = width).
MBCONV_CONFIGS = [
    dict(name=f"M{i}", cin=ci, cout=co, expand=e, k=k, stride=s, hw=h)
    for i, (ci, co, e, k, s, h) in enumerate([
        (32, 16, 1, 3, 1, 112), (16, 24, 6, 3, 2, 112), (24, 24, 6, 3, 1, 56), (24, 40, 6, 5, 2, 56),
        (40, 40, 6, 5, 1, 28), (40, 80, 6, 3, 2, 28), (80, 80, 6, 3, 1, 14), (112, 112, 6, 5, 1, 14),
        (112, 192, 6, 5, 2, 14), (192, 192, 6, 5, 1, 7)])
]


def mbconv_dims(cfg: dict) -> dict:
    """Derived sizes: expanded channels, squeeze width (torchvision: max(1, cin // 4)), output height."""
    exp = cfg["cin"] * cfg["expand"]
    return dict(exp=exp, squeeze=max(1, cfg["cin"] // 4), hw_out=cfg["hw"] // cfg["stride"], pad=cfg["k"] // 2)


def mbconv_input(cfg: dict, seed: int = INPUT_SEED) -> np.ndarray:
    """x [H*W, Cin] fp32 ~ N(0, 1) (NHWC, batch 1)."""
    return normal(seed, (cfg["hw"] * cfg["hw"], cfg["cin"]))


def mbconv_params(cfg: dict) -> dict:
    """Random-init weights of one MBConv block, BatchNorm in inference form (per-channel scale s and
    bias b: y = x * s + b).  1x1 convolutions as [out, in] matrices, the depthwise kernel as one [C]
    vector per tap t = i * k + j; SE as in se_params.  fp32."""
    d = mbconv_dims(cfg)
    cin, cout, exp, S, k = cfg["cin"], cfg["cout"], d["exp"], d["squeeze"], cfg["k"]
    base = 900 + 100 * cfg["k"] + cfg["cin"]
    p = {}
    if cfg["expand"] != 1:
        p.update(We=normal(base + 1, (exp, cin), std=1.0 / np.sqrt(cin)), se=normal(base + 2, (exp,), std=0.1, mean=1.0),
                 be=normal(base + 3, (exp,), std=0.1))
    for t in range(k * k):
        p[f"w{t}"] = normal(base + 10 + t, (exp,), std=1.0 / k)
    p.update(sd=normal(base + 4, (exp,), std=0.1, mean=1.0), bd=normal(base + 5, (exp,), std=0.1),
             W1=normal(base + 6, (S, exp), std=1.0 / np.sqrt(exp)), b1=normal(base + 7, (S,), std=0.02),
             W2=normal(base + 8, (exp, S), std=1.0 / np.sqrt(S)), b2=normal(base + 9, (exp,), std=0.02),
             Wp=normal(base + 40, (cout, exp), std=1.0 / np.sqrt(exp)), sp=normal(base + 41, (cout,), std=0.1, mean=1.0),
             bp=normal(base + 42, (cout,), std=0.1))
    return p


def mbconv_masks(cfg: dict) -> dict:
    """Zero-padding of the depthwise convolution as data: m{t}[h, w] = 1 iff input pixel (h + i - pad,
    w + j - pad) of tap t = i * k + j lies inside the image (a structural constant, like the Swin
    shifted-window mask).  [H, W, 1] fp32 per off-centre tap."""
    H, k, pad = cfg["hw"], cfg["k"], cfg["k"] // 2
    out = {}
    h = np.arange(H)
    for i in range(k):
        for j in range(k):
            if i == pad and j == pad:
                continue
            mh = ((h + i - pad) >= 0) & ((h + i - pad) < H)
            mw = ((h + j - pad) >= 0) & ((h + j - pad) < H)
            out[f"m{i * k + j}"] = (mh[:, None] & mw[None, :]).astype(np.float32).reshape(H, H, 1)
    return out


# ---------------------------------------------------------------- ResNeXt bottleneck blocks R0-R7
# PAPER.md Table 2 (L1303): ResNeXt-101 with 64 groups x 4d bottleneck width (torchvision
# resnext101_64x4d: groups 64, width_per_group 4, layers [3, 4, 23, 3], stride on the grouped 3x3
# convolution).  Its distinct Bottleneck shapes: the first block of each stage (projection shortcut,
# stride 2 from stage 2 on) and the repeated identity block, batch 1, NHWC.
RESNEXT_CONFIGS = [
    dict(name=f"R{i}", cin=ci, width=w, cout=co, hw=h, stride=s, groups=64)
    for i, (ci, w, co, h, s) in enumerate([
        (64, 256, 256, 56, 1), (256, 256, 256, 56, 1), (256, 512, 512, 56, 2), (512, 512, 512, 28, 1),
        (512, 1024, 1024, 28, 2), (1024, 1024, 1024, 14, 1), (1024, 2048, 2048, 14, 2), (2048, 2048, 2048, 7, 1)])
]


def resnext_projection(cfg: dict) -> bool:
    """torchvision: a 1x1 (strided) convolution + BN on the shortcut when the shape changes."""
    return cfg["stride"] != 1 or cfg["cin"] != cfg["cout"]


def resnext_input(cfg: dict, seed: int = INPUT_SEED) -> np.ndarray:
    """x [H*W, Cin] fp32 ~ N(0, 1) (NHWC, batch 1)."""
    return normal(seed, (cfg["hw"] * cfg["hw"], cfg["cin"]))


def resnext_params(cfg: dict) -> dict:
    """Random-init weights of one Bottleneck (BatchNorm in inference form: y = x * s + b).  1x1
    convolutions as [out, in] matrices; the grouped 3x3 convolution as one [G, cg_out, cg_in] tensor per
    tap t = i * 3 + j (group g's [cg_out, cg_in] slice of torch's weight[:, :, i, j]); fp32."""
    cin, w, cout, G = cfg["cin"], cfg["width"], cfg["cout"], cfg["groups"]
    cg = w // G
    base = 5000 + cfg["cin"] + 7 * cfg["hw"]
    p = dict(W1=normal(base + 1, (w, cin), std=1.0 / np.sqrt(cin)), s1=normal(base + 2, (w,), std=0.1, mean=1.0),
             b1=normal(base + 3, (w,), std=0.1))
    for t in range(9):
        p[f"W2_{t}"] = normal(base + 10 + t, (G, cg, cg), std=1.0 / np.sqrt(9 * cg))
    p.update(s2=normal(base + 4, (w,), std=0.1, mean=1.0), b2=normal(base + 5, (w,), std=0.1),
             W3=normal(base + 6, (cout, w), std=1.0 / np.sqrt(w)), s3=normal(base + 7, (cout,), std=0.1, mean=1.0),
             b3=normal(base + 8, (cout,), std=0.1))
    if resnext_projection(cfg):
        p.update(Wd=normal(base + 30, (cout, cin), std=1.0 / np.sqrt(cin)), sd=normal(base + 31, (cout,), std=0.1, mean=1.0),
                 bd=normal(base + 32, (cout,), std=0.1))
    return p


def resnext_masks(cfg: dict) -> dict:
    """Zero padding of the 3x3 convolution as data (the border masks of mbconv_masks with k = 3)."""
    return mbconv_masks(dict(hw=cfg["hw"], k=3))
