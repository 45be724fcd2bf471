"""TE-program builders for the evaluated models, through the C ABI (argument marshalling only).

Each builder creates placeholders immediately before their first use -- the same convention as
SURVEY.md Appendix A -- so node ids are a deterministic function of the model.
  bert      BERT encoder, 49 TEs per layer (Table 2; post-LN, erf GELU, eps 1e-12)
  mmoe      multi-gate mixture of experts (Table 2)
  lstm      stacked LSTM, torch.nn.LSTM gate order (Table 2, §8.4)
  fig2      PAPER.md Fig. 2 (L628-633)
  from_spec a plain-data TE program (synth.random_spec format)
"""
from __future__ import annotations

from . import _lib as L

_DT = {"f32": L.F32, "bf16": L.BF16}


def _layernorm(g, x, H, eps, names, gk, bk):
    mu = g.reduce("mean", x, 1)
    d = g.ew("sub", x, mu)
    q = g.ew("mul", d, d)
    v = g.reduce("mean", q, 1)
    ve = g.ew("add_scalar", v, scalar=eps)
    rs = g.ew("rsqrt", ve)
    n = g.ew("mul", d, rs)
    gm = g.placeholder((H,))
    a = g.ew("mul", n, gm)
    be = g.placeholder((H,))
    names[gk], names[bk] = gm, be
    return g.ew("add", a, be)


def bert_layer(g, X, cfg, names):
    S, H, nh, F = cfg["seq"], cfg["hidden"], cfg["heads"], cfg["ffn"]
    d = H // nh
    prec = _DT[cfg["gemm_dtype"]]
    qkv = []
    for nm in ("q", "k", "v"):
        W = g.placeholder((H, H), prec)
        m = g.matmul(X, W, True, prec)
        b = g.placeholder((H,))
        qkv.append(g.ew("add", m, b))
        names["W" + nm], names["b" + nm] = W, b
    Qp, Kp, Vp = [g.permute(g.reshape(t, (S, nh, d)), (1, 0, 2)) for t in qkv]
    Sc = g.matmul(Qp, Kp, True, prec)
    Ss = g.ew("mul_scalar", Sc, scalar=1.0 / (d ** 0.5))
    Mx = g.reduce("max", Ss, 2)
    Sd = g.ew("sub", Ss, Mx)
    E = g.ew("exp", Sd)
    Z = g.reduce("sum", E, 2)
    P = g.ew("div", E, Z)
    Cx = g.matmul(P, Vp, False, prec)
    Cr = g.reshape(g.permute(Cx, (1, 0, 2)), (S, H))
    Wo = g.placeholder((H, H), prec)
    A0 = g.matmul(Cr, Wo, True, prec)
    bo = g.placeholder((H,))
    R1 = g.ew("add", g.ew("add", A0, bo), X)
    L1 = _layernorm(g, R1, H, cfg["eps"], names, "g1", "be1")
    W1 = g.placeholder((F, H), prec)
    F0 = g.matmul(L1, W1, True, prec)
    c1 = g.placeholder((F,))
    F2 = g.ew("gelu_erf", g.ew("add", F0, c1))
    W2 = g.placeholder((H, F), prec)
    O0 = g.matmul(F2, W2, True, prec)
    c2 = g.placeholder((H,))
    R2 = g.ew("add", g.ew("add", O0, c2), L1)
    names.update(Wo=Wo, bo=bo, W1=W1, c1=c1, W2=W2, c2=c2)
    return _layernorm(g, R2, H, cfg["eps"], names, "g2", "be2")


def bert(cfg, layers=None):
    """Returns (graph, X id, [per-layer name->id], output id)."""
    g = L.Graph()
    X = g.placeholder((cfg["seq"], cfg["hidden"]), L.F32, const=False)
    plist = []
    h = X
    for _ in range(cfg["layers"] if layers is None else layers):
        names = {}
        h = bert_layer(g, h, cfg, names)
        plist.append(names)
    g.mark_output(h)
    return g, X, plist, h


def mmoe(cfg):
    D, E, De, T, Th, B = (cfg[k] for k in ("d_in", "experts", "expert_dim", "tasks", "tower_hidden", "batch"))
    wd = _DT[cfg["w_dtype"]]
    g = L.Graph()
    names = {}
    x = g.placeholder((B, D), L.F32, const=False)
    names["x"] = x
    ex = []
    for e in range(E):
        W = g.placeholder((De, D), wd)
        m = g.matmul(x, W, True, L.F32)
        b = g.placeholder((De,))
        ex.append(g.ew("relu", g.ew("add", m, b)))
        names[f"We{e}"], names[f"be{e}"] = W, b
    gates = []
    for k in range(T):
        W = g.placeholder((E, D), wd)
        m = g.matmul(x, W, True, L.F32)
        b = g.placeholder((E,))
        a = g.ew("add", m, b)
        mx = g.reduce("max", a, 1)
        ee = g.ew("exp", g.ew("sub", a, mx))
        z = g.reduce("sum", ee, 1)
        gates.append(g.ew("div", ee, z))
        names[f"Wg{k}"], names[f"bg{k}"] = W, b
    outs = []
    for k in range(T):
        acc = None
        for e in range(E):
            s = g.slice(gates[k], (0, e), (B, e + 1), (1, 1))
            p = g.ew("mul", s, ex[e])
            acc = p if acc is None else g.ew("add", acc, p)
        Wt = g.placeholder((Th, De), wd)
        t0 = g.matmul(acc, Wt, True, L.F32)
        bt = g.placeholder((Th,))
        t2 = g.ew("relu", g.ew("add", t0, bt))
        Wo = g.placeholder((1, Th), wd)
        y0 = g.matmul(t2, Wo, True, L.F32)
        bo = g.placeholder((1,))
        y = g.ew("add", y0, bo)
        g.mark_output(y)
        outs.append(y)
        names[f"Wt{k}"], names[f"bt{k}"], names[f"Wo{k}"], names[f"bo{k}"] = Wt, bt, Wo, bo
    return g, names, outs


def lstm(cfg):
    T, H, I, Ln = cfg["steps"], cfg["hidden"], cfg["input"], cfg["layers"]
    wd = _DT[cfg["w_dtype"]]
    g = L.Graph()
    names = {}
    X = g.placeholder((T, I), L.F32, const=False)
    names["X"] = X
    W, U, bi, bh, h, c = [], [], [], [], [], []
    for n in range(Ln):
        W.append(g.placeholder((4 * H, I if n == 0 else H), wd))
        U.append(g.placeholder((4 * H, H), wd))
        bi.append(g.placeholder((4 * H,)))
        bh.append(g.placeholder((4 * H,)))
        h.append(g.placeholder((1, H), L.F32, const=False))
        c.append(g.placeholder((1, H), L.F32, const=False))
        names.update({f"W{n}": W[n], f"U{n}": U[n], f"bih{n}": bi[n], f"bhh{n}": bh[n], f"h0_{n}": h[n],
                      f"c0_{n}": c[n]})
    top = []
    for t in range(T):
        x = g.slice(X, (t, 0), (t + 1, I), (1, 1))
        for n in range(Ln):
            g1 = g.ew("add", g.matmul(x, W[n], True, L.F32), bi[n])
            g4 = g.ew("add", g.ew("add", g1, g.matmul(h[n], U[n], True, L.F32)), bh[n])
            gi, gf, gg, go = (g.slice(g4, (0, k * H), (1, (k + 1) * H), (1, 1)) for k in range(4))
            i_, f_, g_, o_ = g.ew("sigmoid", gi), g.ew("sigmoid", gf), g.ew("tanh", gg), g.ew("sigmoid", go)
            c[n] = g.ew("add", g.ew("mul", f_, c[n]), g.ew("mul", i_, g_))
            h[n] = g.ew("mul", o_, g.ew("tanh", c[n]))
            x = h[n]
        top.append(x)
        g.mark_output(x)
    for n in range(Ln):
        g.mark_output(h[n])
        g.mark_output(c[n])
    return g, names, top, list(h), list(c)


def fig2():
    g = L.Graph()
    I0 = g.placeholder((64, 64), L.F32, const=False)
    W0 = g.placeholder((64, 64))
    O0 = g.matmul(I0, W0, False)
    O1 = g.ew("sigmoid", O0)
    W2 = g.placeholder((64, 64))
    O2 = g.matmul(O1, W2, False)
    O3 = g.ew("add", O0, O2)
    W4 = g.placeholder((64, 256))
    O4 = g.matmul(O3, W4, False)
    g.mark_output(O4)
    return g, dict(TE0=O0, TE1=O1, TE2=O2, TE3=O3, TE4=O4)


def from_spec(spec):
    """Build a graph from the plain-data spec format documented in synth/__init__.py."""
    g = L.Graph()
    for n in spec["nodes"]:
        op = n["op"]
        if op == "placeholder":
            g.placeholder(n["shape"], _DT[n["dtype"]], bool(n["const"]))
        elif op == "matmul":
            g.matmul(n["a"], n["b"], bool(n["trans_b"]), _DT[n["prec"]])
        elif op == "ew":
            g.ew(n["fn"], *n["in"], scalar=n.get("scalar", 0.0))
        elif op == "reduce":
            g.reduce(n["fn"], n["in"], n["axis"], bool(n["keepdim"]))
        elif op == "reshape":
            g.reshape(n["in"], n["shape"])
        elif op == "permute":
            g.permute(n["in"], n["perm"])
        elif op == "slice":
            g.slice(n["in"], n["begin"], n["end"], n["stride"])
        else:
            raise ValueError(op)
    for o in spec["outputs"]:
        g.mark_output(o)
    return g


# ---------------------------------------------------------------- Swin-Transformer (Table 2)
def _swin_res(cfg, i):
    return cfg["image"] // cfg["patch"] // (2 ** i)


def _swin_shift(cfg, i, j):
    """Odd blocks use shifted windows (w // 2) unless the window already covers the whole map."""
    w = cfg["window"]
    return 0 if (j % 2 == 0 or w >= _swin_res(cfg, i)) else w // 2


def _swin_block(g, x, cfg, B, R, C, nh, shift, gb, names):
    """x [B*R*R, C] -> x + proj(W-MSA / SW-MSA(LN1 x)) -> + MLP(LN2 x).  The cyclic shift is a roll
    TE and the window partition / reverse are reshape + permute TEs: all one-relies-on-one index
    maps that the lowering folds into the neighbouring GEMM loads and stores (§6.2)."""
    w = cfg["window"]
    n = R // w
    nW, L2 = n * n, w * w
    d = C // nh
    prec = _DT[cfg["gemm_dtype"]]
    pre = f"b{gb}."
    h = _layernorm(g, x, C, cfg["eps"], names, pre + "g1", pre + "be1")
    t = g.reshape(h, (B, R, R, C))
    if shift:
        t = g.roll(t, (0, -shift, -shift, 0))
    t = g.reshape(g.permute(g.reshape(t, (B, n, w, n, w, C)), (0, 1, 3, 2, 4, 5)), (B * nW * L2, C))
    Wqkv = g.placeholder((3 * C, C), prec)
    qkv = g.matmul(t, Wqkv, True, prec)
    bqkv = g.placeholder((3 * C,))
    qkv = g.ew("add", qkv, bqkv)
    names[pre + "Wqkv"], names[pre + "bqkv"] = Wqkv, bqkv
    qkv = g.permute(g.reshape(qkv, (B * nW, L2, 3, nh, d)), (2, 0, 3, 1, 4))
    q, k, v = [g.reshape(g.slice(qkv, (j, 0, 0, 0, 0), (j + 1, B * nW, nh, L2, d), (1, 1, 1, 1, 1)), (B * nW, nh, L2, d))
               for j in range(3)]
    q = g.ew("mul_scalar", q, scalar=float(d) ** -0.5)
    a = g.matmul(q, k, True, prec)
    bias = g.placeholder((nh, L2, L2))
    names[pre + "bias"] = bias
    a = g.ew("add", a, bias)
    if shift:
        a = g.reshape(a, (B, nW, nh, L2, L2))
        mask = g.placeholder((nW, 1, L2, L2))
        names[pre + "mask"] = mask
        a = g.reshape(g.ew("add", a, mask), (B * nW, nh, L2, L2))
    mx = g.reduce("max", a, 3)
    e = g.ew("exp", g.ew("sub", a, mx))
    z = g.reduce("sum", e, 3)
    p = g.ew("div", e, z)
    o = g.matmul(p, v, False, prec)
    o = g.reshape(g.permute(o, (0, 2, 1, 3)), (B * nW * L2, C))
    Wp = g.placeholder((C, C), prec)
    o = g.matmul(o, Wp, True, prec)
    bp = g.placeholder((C,))
    o = g.ew("add", o, bp)
    names[pre + "Wproj"], names[pre + "bproj"] = Wp, bp
    o = g.reshape(g.permute(g.reshape(o, (B, n, n, w, w, C)), (0, 1, 3, 2, 4, 5)), (B, R, R, C))
    if shift:
        o = g.roll(o, (0, shift, shift, 0))
    x = g.ew("add", x, g.reshape(o, (B * R * R, C)))
    h = _layernorm(g, x, C, cfg["eps"], names, pre + "g2", pre + "be2")
    F = cfg["mlp_ratio"] * C
    W1 = g.placeholder((F, C), prec)
    f = g.matmul(h, W1, True, prec)
    b1 = g.placeholder((F,))
    f = g.ew("gelu_erf", g.ew("add", f, b1))
    W2 = g.placeholder((C, F), prec)
    f = g.matmul(f, W2, True, prec)
    b2 = g.placeholder((C,))
    f = g.ew("add", f, b2)
    names.update({pre + "W1": W1, pre + "b1": b1, pre + "W2": W2, pre + "b2": b2})
    return g.ew("add", x, f)


def swin(cfg):
    """Swin-Transformer (torchvision SwinTransformer v1 semantics).  Returns (graph, names, image id,
    logits id); `names` maps every other placeholder to the key used by synth.swin.swin_feed_values."""
    g = L.Graph()
    names = {}
    B, p, C, img = cfg["batch"], cfg["patch"], cfg["embed"], cfg["image"]
    prec = _DT[cfg["gemm_dtype"]]
    R = img // p
    x = g.placeholder((B, 3, img, img), L.F32, const=False)
    # patch embedding: Conv2d(3, C, p, stride p) = im2col (reshape + permute) + GEMM
    t = g.reshape(g.permute(g.reshape(x, (B, 3, R, p, R, p)), (0, 2, 4, 1, 3, 5)), (B * R * R, 3 * p * p))
    Wpe = g.placeholder((C, 3 * p * p), prec)
    t = g.matmul(t, Wpe, True, prec)
    bpe = g.placeholder((C,))
    t = g.ew("add", t, bpe)
    names["Wpe"], names["bpe"] = Wpe, bpe
    h = _layernorm(g, t, C, cfg["eps"], names, "gpe", "bepe")
    gb = 0
    for i, (depth, nh) in enumerate(zip(cfg["depths"], cfg["heads"])):
        R = _swin_res(cfg, i)
        for j in range(depth):
            h = _swin_block(g, h, cfg, B, R, C, nh, _swin_shift(cfg, i, j), gb, names)
            gb += 1
        if i < len(cfg["depths"]) - 1:
            # patch merging: channel blocks (h even, w even), (odd, even), (even, odd), (odd, odd)
            t = g.reshape(g.permute(g.reshape(h, (B, R // 2, 2, R // 2, 2, C)), (0, 1, 3, 4, 2, 5)),
                          (B * (R // 2) ** 2, 4 * C))
            t = _layernorm(g, t, 4 * C, cfg["eps"], names, f"m{i}.g", f"m{i}.be")
            Wm = g.placeholder((2 * C, 4 * C), prec)
            h = g.matmul(t, Wm, True, prec)
            names[f"m{i}.W"] = Wm
            C *= 2
    R = _swin_res(cfg, len(cfg["depths"]) - 1)
    h = _layernorm(g, h, C, cfg["eps"], names, "gn", "ben")
    h = g.reduce("mean", g.reshape(h, (B, R * R, C)), 1, False)
    Wh = g.placeholder((cfg["classes"], C), prec)
    y = g.matmul(h, Wh, True, prec)
    bh = g.placeholder((cfg["classes"],))
    y = g.ew("add", y, bh)
    names["Wh"], names["bh"] = Wh, bh
    g.mark_output(y)
    return g, names, x, y


# ---------------------------------------------------------------- EfficientNet SE sub-module (Fig. 5)
def se_module(cfg):
    """y = x * sigmoid(fc2(silu(fc1(mean_rows(x))))), x [H*W, C] (same node order as oracle.graphs)."""
    HW, C, S = cfg["hw"] * cfg["hw"], cfg["channels"], cfg["squeeze"]
    g = L.Graph()
    x = g.placeholder((HW, C), L.F32, const=False)
    p = g.reduce("mean", x, 0, True)
    W1 = g.placeholder((S, C))
    h = g.matmul(p, W1, True, L.F32)
    b1 = g.placeholder((S,))
    h = g.ew("add", h, b1)
    h = g.ew("mul", h, g.ew("sigmoid", h))
    W2 = g.placeholder((C, S))
    gt = g.matmul(h, W2, True, L.F32)
    b2 = g.placeholder((C,))
    gt = g.ew("sigmoid", g.ew("add", gt, b2))
    y = g.ew("mul", x, gt)
    g.mark_output(y)
    return g, dict(x=x, W1=W1, b1=b1, W2=W2, b2=b2), x, y


def mbconv(cfg):
    """EfficientNet MBConv block as a TE program (same node order as oracle.graphs.mbconv): 1x1
    convolutions as matmuls, the depthwise convolution as rolled, border-masked and weighted taps,
    squeeze-and-excitation, BatchNorm as a per-channel affine; x [H*W, Cin] NHWC, batch 1."""
    H, k, s, pad = cfg["hw"], cfg["k"], cfg["stride"], cfg["k"] // 2
    cin, cout = cfg["cin"], cfg["cout"]
    exp, S = cin * cfg["expand"], max(1, cin // 4)
    Ho = H // s
    g = L.Graph()
    names = {}
    x = g.placeholder((H * H, cin), L.F32, const=False)
    a = x
    if cfg["expand"] != 1:
        names["We"] = g.placeholder((exp, cin))
        a = g.matmul(x, names["We"], True, L.F32)
        names["se"], names["be"] = g.placeholder((exp,)), g.placeholder((exp,))
        a = g.ew("add", g.ew("mul", a, names["se"]), names["be"])
        a = g.ew("mul", a, g.ew("sigmoid", a))
    a3 = g.reshape(a, (H, H, exp))
    acc = None
    for i in range(k):
        for j in range(k):
            t = i * k + j
            if i == pad and j == pad:
                term = a3
            else:
                r = g.roll(a3, (pad - i, pad - j, 0))
                names[f"m{t}"] = g.placeholder((H, H, 1))
                term = g.ew("mul", r, names[f"m{t}"])
            names[f"w{t}"] = g.placeholder((exp,))
            term = g.ew("mul", term, names[f"w{t}"])
            acc = term if acc is None else g.ew("add", acc, term)
    if s != 1:
        acc = g.slice(acc, (0, 0, 0), (H, H, exp), (s, s, 1))
    d = g.reshape(acc, (Ho * Ho, exp))
    names["sd"], names["bd"] = g.placeholder((exp,)), g.placeholder((exp,))
    d = g.ew("add", g.ew("mul", d, names["sd"]), names["bd"])
    d = g.ew("mul", d, g.ew("sigmoid", d))
    p = g.reduce("mean", d, 0, True)
    names["W1"] = g.placeholder((S, exp))
    h = g.matmul(p, names["W1"], True, L.F32)
    names["b1"] = g.placeholder((S,))
    h = g.ew("add", h, names["b1"])
    h = g.ew("mul", h, g.ew("sigmoid", h))
    names["W2"] = g.placeholder((exp, S))
    gt = g.matmul(h, names["W2"], True, L.F32)
    names["b2"] = g.placeholder((exp,))
    gt = g.ew("sigmoid", g.ew("add", gt, names["b2"]))
    d = g.ew("mul", d, gt)
    names["Wp"] = g.placeholder((cout, exp))
    y = g.matmul(d, names["Wp"], True, L.F32)
    names["sp"], names["bp"] = g.placeholder((cout,)), g.placeholder((cout,))
    y = g.ew("add", g.ew("mul", y, names["sp"]), names["bp"])
    if s == 1 and cin == cout:
        y = g.ew("add", y, x)
    g.mark_output(y)
    return g, names, x, y


def resnext(cfg):
    """ResNeXt Bottleneck block (Table 2: ResNeXt-101, 64 groups x 4d) as a TE program (same
    node order as oracle.graphs.resnext): 1x1 convolutions as matmuls, the grouped 3x3 convolution as
    rolled + border-masked taps, each one batched matmul over the groups; BatchNorm as a per-channel
    affine; x [H*W, Cin] NHWC, batch 1.  Returns (graph, names, x, y)."""
    H, s, G = cfg["hw"], cfg["stride"], cfg["groups"]
    cin, w, cout = cfg["cin"], cfg["width"], cfg["cout"]
    cg, Ho = w // G, H // s
    g = L.Graph()
    names = {}
    x = g.placeholder((H * H, cin), L.F32, const=False)
    names["W1"] = g.placeholder((w, cin))
    a = g.matmul(x, names["W1"], True, L.F32)
    names["s1"], names["b1"] = g.placeholder((w,)), g.placeholder((w,))
    a = g.ew("relu", g.ew("add", g.ew("mul", a, names["s1"]), names["b1"]))
    a3 = g.reshape(a, (H, H, w))
    acc = None
    for i in range(3):
        for j in range(3):
            t = i * 3 + j
            if i == 1 and j == 1:
                term = a3
            else:
                r = g.roll(a3, (1 - i, 1 - j, 0))
                names[f"m{t}"] = g.placeholder((H, H, 1))
                term = g.ew("mul", r, names[f"m{t}"])
            tg = g.permute(g.reshape(term, (H * H, G, cg)), (1, 0, 2))
            names[f"W2_{t}"] = g.placeholder((G, cg, cg))
            pt = g.matmul(tg, names[f"W2_{t}"], True, L.F32)
            acc = pt if acc is None else g.ew("add", acc, pt)
    c3 = g.reshape(g.permute(acc, (1, 0, 2)), (H, H, w))
    if s != 1:
        c3 = g.slice(c3, (0, 0, 0), (H, H, w), (s, s, 1))
    d = g.reshape(c3, (Ho * Ho, w))
    names["s2"], names["b2"] = g.placeholder((w,)), g.placeholder((w,))
    d = g.ew("relu", g.ew("add", g.ew("mul", d, names["s2"]), names["b2"]))
    names["W3"] = g.placeholder((cout, w))
    y = g.matmul(d, names["W3"], True, L.F32)
    names["s3"], names["b3"] = g.placeholder((cout,)), g.placeholder((cout,))
    y = g.ew("add", g.ew("mul", y, names["s3"]), names["b3"])
    if s != 1 or cin != cout:
        xs = x
        if s != 1:
            xs = g.reshape(g.slice(g.reshape(x, (H, H, cin)), (0, 0, 0), (H, H, cin), (s, s, 1)), (Ho * Ho, cin))
        names["Wd"] = g.placeholder((cout, cin))
        sc = g.matmul(xs, names["Wd"], True, L.F32)
        names["sd"], names["bd"] = g.placeholder((cout,)), g.placeholder((cout,))
        sc = g.ew("add", g.ew("mul", sc, names["sd"]), names["bd"])
    else:
        sc = x
    y = g.ew("relu", g.ew("add", y, sc))
    g.mark_output(y)
    return g, names, x, y
