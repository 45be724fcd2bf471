"""Oracle-own TE-program builders (TEST INFRASTRUCTURE ONLY; see oracle/te.py header).

The canonical programs follow SURVEY.md Appendix A (a restatement of the paper's models):
  fig2()   PAPER.md Fig. 2 L628-633 (TE4 reads O3: the printed O4[i,rk] self-reference is a garble)
  fig3()   PAPER.md Fig. 3 L970-982 (two GEMMs, horizontal transformation)
  fig4()   PAPER.md Fig. 4 L1030-1050 (relu -> strided slice -> permute, vertical transformation)
  bert()   BERT encoder (Table 2): 49 TEs per layer, post-LN, exact-erf GELU, eps 1e-12
  mmoe()   MMoE (Table 2, ref [32]): 8 experts, 2 gates, 2 towers (sizes are a reading)
  lstm()   stacked LSTM (Table 2, §8.4): torch.nn.LSTM semantics

Placeholders are created immediately before their first use, so node ids are a deterministic
function of the model; the product-side builder follows the same convention and the tests check
that both produce the same node sequence.
"""
from __future__ import annotations


class SpecBuilder:
    def __init__(self):
        self.nodes = []
        self.outputs = []

    def _add(self, n):
        self.nodes.append(n)
        return len(self.nodes) - 1

    def ph(self, shape, dtype="f32", const=1):
        return self._add(dict(op="placeholder", shape=list(shape), dtype=dtype, const=const))

    def mm(self, a, b, trans_b=1, prec="f32"):
        return self._add(dict(op="matmul", a=a, b=b, trans_b=trans_b, prec=prec))

    def ew(self, fn, *ins, scalar=0.0):
        return self._add({"op": "ew", "fn": fn, "in": list(ins), "scalar": float(scalar)})

    def red(self, fn, x, axis, keepdim=1):
        return self._add({"op": "reduce", "fn": fn, "in": x, "axis": axis, "keepdim": keepdim})

    def reshape(self, x, shape):
        return self._add({"op": "reshape", "in": x, "shape": list(shape)})

    def permute(self, x, perm):
        return self._add({"op": "permute", "in": x, "perm": list(perm)})

    def slice(self, x, begin, end, stride):
        return self._add({"op": "slice", "in": x, "begin": list(begin), "end": list(end), "stride": list(stride)})

    def out(self, t):
        self.outputs.append(t)

    def spec(self):
        return {"nodes": self.nodes, "outputs": list(self.outputs)}


def fig2():
    b = SpecBuilder()
    I0 = b.ph((64, 64), const=0)
    W0 = b.ph((64, 64))
    O0 = b.mm(I0, W0, trans_b=0)          # TE0
    O1 = b.ew("sigmoid", O0)              # TE1
    W2 = b.ph((64, 64))
    O2 = b.mm(O1, W2, trans_b=0)          # TE2
    O3 = b.ew("add", O0, O2)              # TE3
    W4 = b.ph((64, 256))
    O4 = b.mm(O3, W4, trans_b=0)          # TE4
    b.out(O4)
    return b.spec(), dict(TE0=O0, TE1=O1, TE2=O2, TE3=O3, TE4=O4)


def fig3():
    b = SpecBuilder()
    A1 = b.ph((4, 8), const=0)
    B1 = b.ph((8, 16))
    C1 = b.mm(A1, B1, trans_b=0)
    A2 = b.ph((2, 8), const=0)
    B2 = b.ph((8, 16))
    C2 = b.mm(A2, B2, trans_b=0)
    b.out(C1)
    b.out(C2)
    return b.spec(), dict(C1=C1, C2=C2, A1=A1, B1=B1, A2=A2, B2=B2)


def fig4():
    b = SpecBuilder()
    A = b.ph((4, 8), const=0)
    B = b.ew("relu", A)
    C = b.slice(B, (0, 0), (4, 4), (2, 1))   # C[i,j] = B[2i, j], shape (2,4)
    D = b.permute(C, (1, 0))                 # D[i,j] = C[j,i], shape (4,2)
    b.out(D)
    return b.spec(), dict(A=A, B=B, C=C, D=D)


def _layernorm(b, x, H, eps, prefix_gamma, prefix_beta):
    mu = b.red("mean", x, 1)
    d = b.ew("sub", x, mu)
    q = b.ew("mul", d, d)
    v = b.red("mean", q, 1)
    ve = b.ew("add_scalar", v, scalar=eps)
    rs = b.ew("rsqrt", ve)
    nrm = b.ew("mul", d, rs)
    g = b.ph((H,))
    gm = b.ew("mul", nrm, g)
    be = b.ph((H,))
    return b.ew("add", gm, be), (g, be)


def bert_layer(b, X, cfg, params):
    """Append one post-LN BERT encoder layer (49 TEs) to builder b.  params collects
    placeholder ids by name."""
    S, H, nh, F = cfg["seq"], cfg["hidden"], cfg["heads"], cfg["ffn"]
    d = H // nh
    prec = cfg["gemm_dtype"]
    wd = cfg["gemm_dtype"]
    qkv = []
    for nm in ("q", "k", "v"):
        W = b.ph((H, H), dtype=wd)
        m0 = b.mm(X, W, 1, prec)
        bb = b.ph((H,))
        m1 = b.ew("add", m0, bb)
        params["W" + nm], params["b" + nm] = W, bb
        qkv.append(m1)
    heads = []
    for m1 in qkv:
        r = b.reshape(m1, (S, nh, d))
        heads.append(b.permute(r, (1, 0, 2)))
    Qp, Kp, Vp = heads
    Sc = b.mm(Qp, Kp, 1, prec)
    Ss = b.ew("mul_scalar", Sc, scalar=1.0 / (d ** 0.5))
    Mx = b.red("max", Ss, 2)
    Sd = b.ew("sub", Ss, Mx)
    E = b.ew("exp", Sd)
    Z = b.red("sum", E, 2)
    P = b.ew("div", E, Z)
    Cx = b.mm(P, Vp, 0, prec)
    Ct = b.permute(Cx, (1, 0, 2))
    Cr = b.reshape(Ct, (S, H))
    Wo = b.ph((H, H), dtype=wd)
    A0 = b.mm(Cr, Wo, 1, prec)
    bo = b.ph((H,))
    A1 = b.ew("add", A0, bo)
    R1 = b.ew("add", A1, X)
    L1, (g1, be1) = _layernorm(b, R1, H, cfg["eps"], "g1", "be1")
    W1 = b.ph((F, H), dtype=wd)
    F0 = b.mm(L1, W1, 1, prec)
    c1 = b.ph((F,))
    F1 = b.ew("add", F0, c1)
    F2 = b.ew("gelu_erf", F1)
    W2 = b.ph((H, F), dtype=wd)
    O0 = b.mm(F2, W2, 1, prec)
    c2 = b.ph((H,))
    O1 = b.ew("add", O0, c2)
    R2 = b.ew("add", O1, L1)
    Y, (g2, be2) = _layernorm(b, R2, H, cfg["eps"], "g2", "be2")
    params.update(Wo=Wo, bo=bo, g1=g1, be1=be1, W1=W1, c1=c1, W2=W2, c2=c2, g2=g2, be2=be2)
    return Y


def bert(cfg, layers=None):
    """BERT encoder over the post-embedding hidden state X [S, H].  Returns (spec, X id, list of
    per-layer param-id dicts, output id)."""
    b = SpecBuilder()
    X = b.ph((cfg["seq"], cfg["hidden"]), const=0)
    plist = []
    h = X
    for _ in range(layers if layers is not None else cfg["layers"]):
        p = {}
        h = bert_layer(b, h, cfg, p)
        plist.append(p)
    b.out(h)
    return b.spec(), X, plist, h


def bert_feed(X_id, plist, x, weights):
    """Map placeholder ids -> stored arrays for bert()."""
    feed = {X_id: x}
    for p, w in zip(plist, weights):
        for k, i in p.items():
            feed[i] = w[k]
    return feed


def mmoe(cfg):
    D, E, De, T, Th = cfg["d_in"], cfg["experts"], cfg["expert_dim"], cfg["tasks"], cfg["tower_hidden"]
    B = cfg["batch"]
    wd = cfg["w_dtype"]
    b = SpecBuilder()
    names = {}
    x = b.ph((B, D), const=0)
    names["x"] = x
    ex = []
    for e in range(E):
        W = b.ph((De, D), dtype=wd)
        m = b.mm(x, W, 1, "f32")
        bb = b.ph((De,))
        a = b.ew("add", m, bb)
        ex.append(b.ew("relu", a))
        names[f"We{e}"], names[f"be{e}"] = W, bb
    gates = []
    for k in range(T):
        W = b.ph((E, D), dtype=wd)
        m = b.mm(x, W, 1, "f32")
        bb = b.ph((E,))
        a = b.ew("add", m, bb)
        mx = b.red("max", a, 1)
        sd = b.ew("sub", a, mx)
        ee = b.ew("exp", sd)
        z = b.red("sum", ee, 1)
        gates.append(b.ew("div", ee, z))
        names[f"Wg{k}"], names[f"bg{k}"] = W, bb
    outs = []
    for k in range(T):
        acc = None
        for e in range(E):
            s = b.slice(gates[k], (0, e), (B, e + 1), (1, 1))
            p = b.ew("mul", s, ex[e])
            acc = p if acc is None else b.ew("add", acc, p)
        Wt = b.ph((Th, De), dtype=wd)
        t0 = b.mm(acc, Wt, 1, "f32")
        bt = b.ph((Th,))
        t1 = b.ew("add", t0, bt)
        t2 = b.ew("relu", t1)
        Wo = b.ph((1, Th), dtype=wd)
        y0 = b.mm(t2, Wo, 1, "f32")
        bo = b.ph((1,))
        y1 = b.ew("add", y0, bo)
        b.out(y1)
        outs.append(y1)
        names[f"Wt{k}"], names[f"bt{k}"], names[f"Wo{k}"], names[f"bo{k}"] = Wt, bt, Wo, bo
    return b.spec(), names, outs


def lstm(cfg):
    """Stacked LSTM, torch.nn.LSTM gate order i, f, g, o; h0 = c0 = 0 supplied as placeholders.
    Per cell-step: 2 GEMVs + 3 adds + 4 slices + 4 activations + 5 state ops."""
    T, H, I, L = cfg["steps"], cfg["hidden"], cfg["input"], cfg["layers"]
    wd = cfg["w_dtype"]
    b = SpecBuilder()
    names = {}
    X = b.ph((T, I), const=0)
    names["X"] = X
    W, U, bi, bh, h, c = [], [], [], [], [], []
    for n in range(L):
        W.append(b.ph((4 * H, I if n == 0 else H), dtype=wd))
        U.append(b.ph((4 * H, H), dtype=wd))
        bi.append(b.ph((4 * H,)))
        bh.append(b.ph((4 * H,)))
        h.append(b.ph((1, H), const=0))
        c.append(b.ph((1, H), const=0))
        names.update({f"W{n}": W[n], f"U{n}": U[n], f"bih{n}": bi[n], f"bhh{n}": bh[n], f"h0_{n}": h[n],
                      f"c0_{n}": c[n]})
    top = []
    for t in range(T):
        x = b.slice(X, (t, 0), (t + 1, I), (1, 1))
        for n in range(L):
            g0 = b.mm(x, W[n], 1, "f32")
            g1 = b.ew("add", g0, bi[n])
            g2 = b.mm(h[n], U[n], 1, "f32")
            g3 = b.ew("add", g1, g2)
            g4 = b.ew("add", g3, bh[n])
            gi = b.slice(g4, (0, 0), (1, H), (1, 1))
            gf = b.slice(g4, (0, H), (1, 2 * H), (1, 1))
            gg = b.slice(g4, (0, 2 * H), (1, 3 * H), (1, 1))
            go = b.slice(g4, (0, 3 * H), (1, 4 * H), (1, 1))
            i_ = b.ew("sigmoid", gi)
            f_ = b.ew("sigmoid", gf)
            g_ = b.ew("tanh", gg)
            o_ = b.ew("sigmoid", go)
            fc = b.ew("mul", f_, c[n])
            ig = b.ew("mul", i_, g_)
            c[n] = b.ew("add", fc, ig)
            tc = b.ew("tanh", c[n])
            h[n] = b.ew("mul", o_, tc)
            x = h[n]
        top.append(x)
        b.out(x)
    for n in range(L):
        b.out(h[n])
        b.out(c[n])
    return b.spec(), names, top, list(h), list(c)


# ---------------------------------------------------------------- Swin-Transformer (Table 2)
def _swin_res(cfg, i):
    return cfg["image"] // cfg["patch"] // (2 ** i)


def _swin_shift(cfg, i, j):
    w = cfg["window"]
    return 0 if (j % 2 == 0 or w >= _swin_res(cfg, i)) else w // 2


def _swin_ln(b, x, C, eps, names, gk, bk):
    out, (g, be) = _layernorm(b, x, C, eps, gk, bk)
    names[gk], names[bk] = g, be
    return out


def swin_block(b, x, cfg, B, R, C, nh, shift, gb, names):
    """One Swin block (pre-LN; W-MSA / SW-MSA then MLP), torchvision `SwinTransformerBlock`:
    x = x + proj(window_attention(LN1(x))); x = x + W2 gelu(W1 LN2(x)).  x is [B*R*R, C] (b, h, w
    row-major).  Cyclic shift = roll TE; window partition / reverse = reshape + permute TEs."""
    w = cfg["window"]
    n = R // w
    nW = n * n
    d = C // nh
    prec = cfg["gemm_dtype"]
    pre = f"b{gb}."
    h = _swin_ln(b, x, C, cfg["eps"], names, pre + "g1", pre + "be1")
    t = b.reshape(h, (B, R, R, C))
    if shift:
        t = b._add({"op": "roll", "in": t, "shifts": [0, -shift, -shift, 0]})
    t = b.reshape(t, (B, n, w, n, w, C))
    t = b.permute(t, (0, 1, 3, 2, 4, 5))
    t = b.reshape(t, (B * nW * w * w, C))
    Wqkv = b.ph((3 * C, C), dtype=prec)
    qkv = b.mm(t, Wqkv, 1, prec)
    bqkv = b.ph((3 * C,))
    qkv = b.ew("add", qkv, bqkv)
    names[pre + "Wqkv"], names[pre + "bqkv"] = Wqkv, bqkv
    qkv = b.reshape(qkv, (B * nW, w * w, 3, nh, d))
    qkv = b.permute(qkv, (2, 0, 3, 1, 4))
    qs, ks, vs = [b.reshape(b.slice(qkv, (k, 0, 0, 0, 0), (k + 1, B * nW, nh, w * w, d), (1, 1, 1, 1, 1)),
                            (B * nW, nh, w * w, d)) for k in range(3)]
    qs = b.ew("mul_scalar", qs, scalar=float(d) ** -0.5)
    a = b.mm(qs, ks, 1, prec)
    bias = b.ph((nh, w * w, w * w))
    names[pre + "bias"] = bias
    a = b.ew("add", a, bias)
    if shift:
        a = b.reshape(a, (B, nW, nh, w * w, w * w))
        mask = b.ph((nW, 1, w * w, w * w))
        names[pre + "mask"] = mask
        a = b.ew("add", a, mask)
        a = b.reshape(a, (B * nW, nh, w * w, w * w))
    mx = b.red("max", a, 3)
    e = b.ew("exp", b.ew("sub", a, mx))
    z = b.red("sum", e, 3)
    p = b.ew("div", e, z)
    o = b.mm(p, vs, 0, prec)
    o = b.reshape(b.permute(o, (0, 2, 1, 3)), (B * nW * w * w, C))
    Wp = b.ph((C, C), dtype=prec)
    o = b.mm(o, Wp, 1, prec)
    bp = b.ph((C,))
    o = b.ew("add", o, bp)
    names[pre + "Wproj"], names[pre + "bproj"] = Wp, bp
    o = b.reshape(o, (B, n, n, w, w, C))
    o = b.permute(o, (0, 1, 3, 2, 4, 5))
    o = b.reshape(o, (B, R, R, C))
    if shift:
        o = b._add({"op": "roll", "in": o, "shifts": [0, shift, shift, 0]})
    o = b.reshape(o, (B * R * R, C))
    x = b.ew("add", x, o)
    h = _swin_ln(b, x, C, cfg["eps"], names, pre + "g2", pre + "be2")
    F = cfg["mlp_ratio"] * C
    W1 = b.ph((F, C), dtype=prec)
    f = b.mm(h, W1, 1, prec)
    b1 = b.ph((F,))
    f = b.ew("gelu_erf", b.ew("add", f, b1))
    W2 = b.ph((C, F), dtype=prec)
    f = b.mm(f, W2, 1, prec)
    b2 = b.ph((C,))
    f = b.ew("add", f, b2)
    names.update({pre + "W1": W1, pre + "b1": b1, pre + "W2": W2, pre + "b2": b2})
    return b.ew("add", x, f)


def swin(cfg):
    """Swin-Transformer (torchvision `SwinTransformer` v1 semantics) as a TE program.
    Returns (spec, names: placeholder name -> id, image id, logits id)."""
    b = SpecBuilder()
    names = {}
    B, p, C = cfg["batch"], cfg["patch"], cfg["embed"]
    prec = cfg["gemm_dtype"]
    img = cfg["image"]
    R = img // p
    x = b.ph((B, 3, img, img), const=0)
    # patch embedding: Conv2d(3, C, p, stride p) == im2col (reshape + permute) + GEMM
    t = b.reshape(x, (B, 3, R, p, R, p))
    t = b.permute(t, (0, 2, 4, 1, 3, 5))
    t = b.reshape(t, (B * R * R, 3 * p * p))
    Wpe = b.ph((C, 3 * p * p), dtype=prec)
    t = b.mm(t, Wpe, 1, prec)
    bpe = b.ph((C,))
    t = b.ew("add", t, bpe)
    names["Wpe"], names["bpe"] = Wpe, bpe
    h = _swin_ln(b, t, C, cfg["eps"], names, "gpe", "bepe")
    gb = 0
    for i, (depth, nh) in enumerate(zip(cfg["depths"], cfg["heads"])):
        R = _swin_res(cfg, i)
        for j in range(depth):
            h = swin_block(b, h, cfg, B, R, C, nh, _swin_shift(cfg, i, j), gb, names)
            gb += 1
        if i < len(cfg["depths"]) - 1:
            # patch merging: cat(x[0::2,0::2], x[1::2,0::2], x[0::2,1::2], x[1::2,1::2]) -> LN -> Linear
            t = b.reshape(h, (B, R // 2, 2, R // 2, 2, C))
            t = b.permute(t, (0, 1, 3, 4, 2, 5))
            t = b.reshape(t, (B * (R // 2) ** 2, 4 * C))
            t = _swin_ln(b, t, 4 * C, cfg["eps"], names, f"m{i}.g", f"m{i}.be")
            Wm = b.ph((2 * C, 4 * C), dtype=prec)
            h = b.mm(t, Wm, 1, prec)
            names[f"m{i}.W"] = Wm
            C *= 2
    R = _swin_res(cfg, len(cfg["depths"]) - 1)
    h = _swin_ln(b, h, C, cfg["eps"], names, "gn", "ben")
    h = b.red("mean", b.reshape(h, (B, R * R, C)), 1, keepdim=0)
    Wh = b.ph((cfg["classes"], C), dtype=prec)
    y = b.mm(h, Wh, 1, prec)
    bh = b.ph((cfg["classes"],))
    y = b.ew("add", y, bh)
    names["Wh"], names["bh"] = Wh, bh
    b.out(y)
    return b.spec(), names, x, y


def se_module(cfg):
    """EfficientNet squeeze-and-excitation sub-module (Fig. 5; torchvision
    SqueezeExcitation with SiLU / Sigmoid): y = x * sigmoid(fc2(silu(fc1(mean_rows(x))))).
    x [H*W, C] (NHWC, batch 1).  Returns (spec, names, x id, y id)."""
    HW, C, S = cfg["hw"] * cfg["hw"], cfg["channels"], cfg["squeeze"]
    b = SpecBuilder()
    x = b.ph((HW, C), const=0)
    p = b.red("mean", x, 0)                    # [1, C] global average pool
    W1 = b.ph((S, C))
    h = b.mm(p, W1, 1, "f32")
    b1 = b.ph((S,))
    h = b.ew("add", h, b1)
    h = b.ew("mul", h, b.ew("sigmoid", h))     # SiLU
    W2 = b.ph((C, S))
    g = b.mm(h, W2, 1, "f32")
    b2 = b.ph((C,))
    g = b.ew("sigmoid", b.ew("add", g, b2))
    y = b.ew("mul", x, g)                      # channel-wise rescale (broadcast over rows)
    b.out(y)
    return b.spec(), dict(x=x, W1=W1, b1=b1, W2=W2, b2=b2), x, y


def mbconv(cfg):
    """EfficientNet MBConv block (the building block of PAPER.md Fig. 5 / 6, L1511-1564; torchvision
    efficientnet_b0 MBConv in inference form) as a TE program over NHWC, batch 1:
      a = SiLU(BN(x W_e^T))                      1x1 expand convolution (omitted when expand == 1)
      d = SiLU(BN(sum_t m_t * roll(a, -o_t) * w_t))[::s, ::s]
                                                  depthwise k x k convolution, zero padding k // 2: tap t
                                                  reads a shifted by its offset o_t (a roll TE) and the
                                                  border mask m_t zeroes what the roll wrapped around
      d = d * sigmoid(fc2(SiLU(fc1(mean(d)))))    squeeze-and-excitation (se_module)
      y = BN(d W_p^T) (+ x when stride 1 and cin == cout)
    BN is the per-channel affine y = x * s + b.  Returns (spec, names, x id, y id)."""
    d_ = synth_dims(cfg)
    H, k, s, pad = cfg["hw"], cfg["k"], cfg["stride"], cfg["k"] // 2
    cin, cout, exp, S = cfg["cin"], cfg["cout"], d_["exp"], d_["squeeze"]
    Ho = H // s
    b = SpecBuilder()
    names = {}
    x = b.ph((H * H, cin), const=0)
    a = x
    if cfg["expand"] != 1:
        names["We"] = b.ph((exp, cin))
        a = b.mm(x, names["We"], 1, "f32")
        names["se"], names["be"] = b.ph((exp,)), b.ph((exp,))
        a = b.ew("add", b.ew("mul", a, names["se"]), names["be"])
        a = b.ew("mul", a, b.ew("sigmoid", a))
    a3 = b.reshape(a, (H, H, exp))
    acc = None
    for i in range(k):
        for j in range(k):
            t = i * k + j
            if i == pad and j == pad:
                term = a3
            else:
                r = b._add({"op": "roll", "in": a3, "shifts": [pad - i, pad - j, 0]})   # r[h, w] = a[h + i - pad, w + j - pad]
                names[f"m{t}"] = b.ph((H, H, 1))
                term = b.ew("mul", r, names[f"m{t}"])
            names[f"w{t}"] = b.ph((exp,))
            term = b.ew("mul", term, names[f"w{t}"])
            acc = term if acc is None else b.ew("add", acc, term)
    if s != 1:
        acc = b.slice(acc, (0, 0, 0), (H, H, exp), (s, s, 1))
    dd = b.reshape(acc, (Ho * Ho, exp))
    names["sd"], names["bd"] = b.ph((exp,)), b.ph((exp,))
    dd = b.ew("add", b.ew("mul", dd, names["sd"]), names["bd"])
    dd = b.ew("mul", dd, b.ew("sigmoid", dd))
    p = b.red("mean", dd, 0)
    names["W1"] = b.ph((S, exp))
    h = b.mm(p, names["W1"], 1, "f32")
    names["b1"] = b.ph((S,))
    h = b.ew("add", h, names["b1"])
    h = b.ew("mul", h, b.ew("sigmoid", h))
    names["W2"] = b.ph((exp, S))
    g = b.mm(h, names["W2"], 1, "f32")
    names["b2"] = b.ph((exp,))
    g = b.ew("sigmoid", b.ew("add", g, names["b2"]))
    dd = b.ew("mul", dd, g)
    names["Wp"] = b.ph((cout, exp))
    y = b.mm(dd, names["Wp"], 1, "f32")
    names["sp"], names["bp"] = b.ph((cout,)), b.ph((cout,))
    y = b.ew("add", b.ew("mul", y, names["sp"]), names["bp"])
    if s == 1 and cin == cout:
        y = b.ew("add", y, x)
    b.out(y)
    return b.spec(), names, x, y


def synth_dims(cfg):
    """exp, squeeze of an MBConv config (torchvision: squeeze = max(1, cin // 4))."""
    return dict(exp=cfg["cin"] * cfg["expand"], squeeze=max(1, cfg["cin"] // 4))


def resnext(cfg):
    """ResNeXt Bottleneck block (Table 2: ResNeXt-101, 64 groups x 4d; torchvision
    resnext101_64x4d Bottleneck in inference form) as a TE program over NHWC, batch 1:
      a = ReLU(BN(x W1^T))                                1x1 convolution to the bottleneck width
      c = sum_t  m_t * roll(a, -o_t)  grouped by G:        the 3x3 grouped convolution, zero padding 1:
          [HW, G, cg] -> [G, HW, cg] (x) W2_t [G, cg, cg]^T  tap t reads a shifted by its offset o_t (a
                                                          roll TE, border mask m_t) and every group g
                                                          multiplies its cg channels by W2_t[g] -- ONE
                                                          batched matmul TE per tap over the G groups
      d = ReLU(BN(c[::s, ::s]))
      y = ReLU(BN(d W3^T) + shortcut),  shortcut = x, or BN(x[::s, ::s] Wd^T) when the shape changes
    BN is the per-channel affine y = x * s + b.  Returns (spec, names, x id, y id)."""
    H, s, G = cfg["hw"], cfg["stride"], cfg["groups"]
    cin, w, cout = cfg["cin"], cfg["width"], cfg["cout"]
    cg, Ho = w // G, H // s
    b = SpecBuilder()
    names = {}
    x = b.ph((H * H, cin), const=0)
    names["W1"] = b.ph((w, cin))
    a = b.mm(x, names["W1"], 1, "f32")
    names["s1"], names["b1"] = b.ph((w,)), b.ph((w,))
    a = b.ew("relu", b.ew("add", b.ew("mul", a, names["s1"]), names["b1"]))
    a3 = b.reshape(a, (H, H, w))
    acc = None
    for i in range(3):
        for j in range(3):
            t = i * 3 + j
            if i == 1 and j == 1:
                term = a3
            else:
                r = b._add({"op": "roll", "in": a3, "shifts": [1 - i, 1 - j, 0]})   # r[h, w] = a[h + i - 1, w + j - 1]
                names[f"m{t}"] = b.ph((H, H, 1))
                term = b.ew("mul", r, names[f"m{t}"])
            tg = b.permute(b.reshape(term, (H * H, G, cg)), (1, 0, 2))           # [G, HW, cg]
            names[f"W2_{t}"] = b.ph((G, cg, cg))
            pt = b.mm(tg, names[f"W2_{t}"], 1, "f32")                             # [G, HW, cg]
            acc = pt if acc is None else b.ew("add", acc, pt)
    c3 = b.reshape(b.permute(acc, (1, 0, 2)), (H, H, w))
    if s != 1:
        c3 = b.slice(c3, (0, 0, 0), (H, H, w), (s, s, 1))
    d = b.reshape(c3, (Ho * Ho, w))
    names["s2"], names["b2"] = b.ph((w,)), b.ph((w,))
    d = b.ew("relu", b.ew("add", b.ew("mul", d, names["s2"]), names["b2"]))
    names["W3"] = b.ph((cout, w))
    y = b.mm(d, names["W3"], 1, "f32")
    names["s3"], names["b3"] = b.ph((cout,)), b.ph((cout,))
    y = b.ew("add", b.ew("mul", y, names["s3"]), names["b3"])
    if s != 1 or cin != cout:
        xs = x
        if s != 1:
            xs = b.reshape(b.slice(b.reshape(x, (H, H, cin)), (0, 0, 0), (H, H, cin), (s, s, 1)), (Ho * Ho, cin))
        names["Wd"] = b.ph((cout, cin))
        sc = b.mm(xs, names["Wd"], 1, "f32")
        names["sd"], names["bd"] = b.ph((cout,)), b.ph((cout,))
        sc = b.ew("add", b.ew("mul", sc, names["sd"]), names["bd"])
    else:
        sc = x
    y = b.ew("relu", b.ew("add", y, sc))
    b.out(y)
    return b.spec(), names, x, y
