"""Pins for the oracle's TE interpreter (CPU only): brute force, closed forms, invariants.

Every check here is independent of the interpreter's own vectorised code path: either the
pure-Python element-by-element definition, a closed form, or a mathematical invariant."""
import math

import numpy as np
import pytest

import synth
from oracle import te
from oracle.graphs import SpecBuilder, bert, bert_feed, fig4


def _rand_int_program(seed):
    spec = synth.random_spec(seed, n_ops=10)
    return spec, synth.spec_inputs(spec, seed, integer=True)


@pytest.mark.parametrize("seed", range(12))
def test_vectorised_equals_brute_force_integer_inputs(seed):
    """Integer-valued inputs on integer-closed ops: both modes must be bit-equal (exact)."""
    b = SpecBuilder()
    r = synth.rng(seed)
    M, K, N = (int(x) for x in r.integers(2, 6, 3))
    a = b.ph((M, K), const=0)
    w = b.ph((N, K))
    w2 = b.ph((K, N))
    m1 = b.mm(a, w, 1)
    m2 = b.mm(a, w2, 0)
    s = b.ew("add", m1, m2)
    c = b.ph((N,))
    t = b.ew("mul", s, c)
    u = b.ew("max", t, m1)
    v = b.ew("sub", u, c)
    rs = b.red("sum", v, 1)
    rm = b.red("max", v, 0, keepdim=0)
    p = b.permute(v, (1, 0))
    rr = b.reshape(p, (N * M,))
    sl = b.slice(p, (0, 1), (N, M), (2, 1))
    bat = b.reshape(v, (1, M, N))
    w3 = b.ph((1, K, N))
    a3 = b.reshape(a, (1, M, K))
    bm = b.mm(a3, w3, 0)
    for o in (rs, rm, rr, sl, bm):
        b.out(o)
    spec = b.spec()
    ins = synth.spec_inputs(spec, seed, integer=True)
    v1 = te.evaluate(spec, ins)
    v2 = te.evaluate(spec, ins, brute=True)
    for x, y in zip(v1, v2):
        assert np.array_equal(x, y)


@pytest.mark.parametrize("seed", range(8))
def test_random_programs_brute_vs_vectorised(seed):
    spec, ins = _rand_int_program(seed)
    ins = synth.spec_inputs(spec, seed)
    v1 = te.evaluate(spec, ins)
    v2 = te.evaluate(spec, ins, brute=True)
    for x, y in zip(v1, v2):
        np.testing.assert_allclose(x, y, rtol=1e-12, atol=1e-12)


def test_bf16_rounding_pins():
    # exactly representable values are fixed points; halfway cases round to even
    assert te.round_bf16(1.0) == 1.0
    assert te.round_bf16(1.0 + 2 ** -8) == 1.0                  # tie -> even mantissa (…0)
    assert te.round_bf16(1.0 + 3 * 2 ** -8) == 1.0 + 2 ** -6     # tie -> even (…10)
    assert te.round_bf16(1.0 + 2 ** -8 + 2 ** -20) == 1.0 + 2 ** -7
    assert te.round_bf16(-3.0) == -3.0
    x = synth.rng(5).standard_normal(1000)
    r = te.round_bf16(x)
    # agreement with the independent bit-level rounding of synth (on fp32-representable inputs)
    x32 = x.astype(np.float32).astype(np.float64)
    np.testing.assert_array_equal(te.round_bf16(x32), synth.to_storage(x32, "bf16").astype(np.float64))
    assert np.all(np.abs(r - x) <= np.abs(x) * 2 ** -8)


def test_softmax_invariants():
    b = SpecBuilder()
    x = b.ph((3, 7), const=0)
    mx = b.red("max", x, 1)
    d = b.ew("sub", x, mx)
    e = b.ew("exp", d)
    z = b.red("sum", e, 1)
    p = b.ew("div", e, z)
    b.out(p)
    spec = b.spec()
    xv = synth.normal(3, (3, 7), std=3.0)
    xv[2, :] = 0.75                         # constant row
    out = te.evaluate(spec, {0: xv})[p]
    np.testing.assert_allclose(out.sum(axis=1), 1.0, atol=1e-12)
    np.testing.assert_allclose(out[2], 1.0 / 7, atol=1e-15)
    shifted = te.evaluate(spec, {0: xv.astype(np.float64) + 11.0})[p]
    np.testing.assert_allclose(shifted, out, atol=1e-12)


def test_layernorm_invariants_and_gelu():
    b = SpecBuilder()
    x = b.ph((4, 16), const=0)
    mu = b.red("mean", x, 1)
    d = b.ew("sub", x, mu)
    q = b.ew("mul", d, d)
    v = b.red("mean", q, 1)
    eps = 1e-3
    ve = b.ew("add_scalar", v, scalar=eps)
    rs = b.ew("rsqrt", ve)
    y = b.ew("mul", d, rs)
    gl = b.ew("gelu_erf", x)
    spec = b.spec()
    xv = synth.normal(4, (4, 16), std=2.0)
    xv[3] = 5.0
    vals = te.evaluate(spec, {0: xv})
    out = vals[y]
    np.testing.assert_allclose(out[:3].mean(axis=1), 0.0, atol=1e-12)
    var_in = xv[:3].astype(np.float64).var(axis=1)
    np.testing.assert_allclose(out[:3].var(axis=1), var_in / (var_in + eps), rtol=1e-12)
    np.testing.assert_array_equal(out[3], 0.0)            # constant row -> 0
    g = vals[gl]
    assert te.unary_scalar("gelu_erf", 0.0) == 0.0
    # gelu(x) - gelu(-x) = x (odd part of x*Phi(x)), a closed-form identity
    xx = xv.astype(np.float64)
    np.testing.assert_allclose(te.unary_vec("gelu_erf", xx) - te.unary_vec("gelu_erf", -xx), xx, atol=1e-12)
    # large positive -> identity, large negative -> 0
    assert abs(te.unary_scalar("gelu_erf", 12.0) - 12.0) < 1e-12 and abs(te.unary_scalar("gelu_erf", -12.0)) < 1e-12


def test_fig4_unfused_values():
    spec, ids = fig4()
    A = synth.normal(9, (4, 8))
    vals = te.evaluate(spec, {ids["A"]: A})
    A64 = A.astype(np.float64)
    for i in range(4):
        for j in range(2):
            assert vals[ids["D"]][i, j] == max(A64[2 * j, i], 0.0)


def test_bert_graph_has_49_tes_per_layer():
    spec, X, plist, y = bert(synth.BERT_TINY, layers=2)
    n_te = sum(1 for n in spec["nodes"] if n["op"] != "placeholder")
    assert n_te == 98
    shapes = te.infer_shapes(spec)
    assert shapes[y] == (32, 64)
