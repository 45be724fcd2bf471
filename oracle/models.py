"""Oracle: direct fp64 formulas of the evaluated models (TEST INFRASTRUCTURE ONLY).

These are the plain definitions the TE programs in graphs.py must reproduce; they are in turn
pinned against torch.nn reference modules in fp64 (tests/test_oracle_models.py).
  bert_layer  post-LN encoder layer (Table 2; readings in DESIGN.md)
  lstm        stacked LSTM, torch.nn.LSTM semantics (Table 2; §8.4)
  mmoe        multi-gate mixture of experts (Table 2, ref [32] L2138-2142)
  fig2        PAPER.md Fig. 2
"""
from __future__ import annotations

import numpy as np
from scipy.special import erf

from .te import round_bf16


def _f64(x):
    return np.asarray(x, dtype=np.float64)


def _ln(x, g, b, eps):
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps) * g + b


def _mm(a, b, bf16):
    if bf16:
        a, b = round_bf16(a), round_bf16(b)
    return a @ b


def bert_layer(x, p, heads, eps=1e-12, bf16_operands=False):
    x = _f64(x)
    p = {k: _f64(v) for k, v in p.items()}
    S, H = x.shape
    d = H // heads
    q = _mm(x, p["Wq"].T, bf16_operands) + p["bq"]
    k = _mm(x, p["Wk"].T, bf16_operands) + p["bk"]
    v = _mm(x, p["Wv"].T, bf16_operands) + p["bv"]
    sp = lambda t: t.reshape(S, heads, d).transpose(1, 0, 2)
    q, k, v = sp(q), sp(k), sp(v)
    s = _mm(q, k.transpose(0, 2, 1), bf16_operands) / np.sqrt(d)
    s = np.exp(s - s.max(axis=-1, keepdims=True))
    pr = s / s.sum(axis=-1, keepdims=True)
    ctx = _mm(pr, v, bf16_operands).transpose(1, 0, 2).reshape(S, H)
    a = _mm(ctx, p["Wo"].T, bf16_operands) + p["bo"] + x
    l1 = _ln(a, p["g1"], p["be1"], eps)
    f = _mm(l1, p["W1"].T, bf16_operands) + p["c1"]
    f = 0.5 * f * (1.0 + erf(f / np.sqrt(2.0)))
    o = _mm(f, p["W2"].T, bf16_operands) + p["c2"] + l1
    return _ln(o, p["g2"], p["be2"], eps)


def bert(x, weights, heads, eps=1e-12, bf16_operands=False):
    h = _f64(x)
    for p in weights:
        h = bert_layer(h, p, heads, eps, bf16_operands)
    return h


def _sig(z):
    return 1.0 / (1.0 + np.exp(-z))


def lstm(x, params, H):
    """Returns (top-layer h for every step [T,H], final h per layer, final c per layer)."""
    x = _f64(x)
    T = x.shape[0]
    L = len(params)
    h = [np.zeros(H) for _ in range(L)]
    c = [np.zeros(H) for _ in range(L)]
    top = np.zeros((T, H))
    for t in range(T):
        inp = x[t]
        for n, p in enumerate(params):
            g = _f64(p["W"]) @ inp + _f64(p["b_ih"]) + _f64(p["U"]) @ h[n] + _f64(p["b_hh"])
            i, f, gg, o = _sig(g[:H]), _sig(g[H:2 * H]), np.tanh(g[2 * H:3 * H]), _sig(g[3 * H:])
            c[n] = f * c[n] + i * gg
            h[n] = o * np.tanh(c[n])
            inp = h[n]
        top[t] = inp
    return top, h, c


def mmoe(x, p, cfg):
    x = _f64(x)
    E, T = cfg["experts"], cfg["tasks"]
    ex = [np.maximum(x @ _f64(p[f"We{e}"]).T + _f64(p[f"be{e}"]), 0.0) for e in range(E)]
    ys = []
    for k in range(T):
        z = x @ _f64(p[f"Wg{k}"]).T + _f64(p[f"bg{k}"])
        g = np.exp(z - z.max(axis=1, keepdims=True))
        g = g / g.sum(axis=1, keepdims=True)
        f = sum(g[:, e:e + 1] * ex[e] for e in range(E))
        t = np.maximum(f @ _f64(p[f"Wt{k}"]).T + _f64(p[f"bt{k}"]), 0.0)
        ys.append(t @ _f64(p[f"Wo{k}"]).T + _f64(p[f"bo{k}"]))
    return ys


def fig2(I0, W0, W2, W4):
    I0, W0, W2, W4 = map(_f64, (I0, W0, W2, W4))
    O0 = I0 @ W0
    O1 = _sig(O0)
    O2 = O1 @ W2
    O3 = O0 + O2
    return O3 @ W4
