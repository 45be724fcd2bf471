"""GPU: single stages of the persistent BERT kernel (kernels/bert.cu) in isolation, bit-exact on
integer inputs, and the LayerNorm row stage on degenerate rows.

Stage isolation: SOUFFLE_BERT_STAGES=b,e runs only stages [b, e) of the stage list (stage 0 converts
the input, then 6 per layer: QKV, attention + out-projection, LN1, FFN1, FFN2, LN2); the test reads
the kernel's workspace buffers through souffle_plan_debug_region.  Inputs in {-2..2}: every product
and partial sum is an integer below 2^24, exact in bf16 operands and fp32 accumulation, so the GEMM
stages (TMA K-chunk rotation, 128-byte swizzle, tcgen05 tiles, head-major / V^T scatter stores,
split-K partials) must reproduce the integer GEMM bit for bit (bf16 outputs: RNE of the exact
integer)."""
import os

import numpy as np
import pytest
import torch

import synth
from oracle import graphs as og
from oracle import te
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L
from paper_conf_asplos_xiazswwyfc24_b200 import models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session

pytestmark = pytest.mark.gpu
CFG = dict(synth.BERT_BASE, layers=1)


def _bf16_rne(a):
    """fp64 -> bf16 (RNE) -> fp64 through torch's conversion (not the kernel)."""
    return torch.from_numpy(np.asarray(a, np.float64)).to(torch.bfloat16).double().numpy()


def _session(cfg, w, x):
    g, gX, gpl, gy = M.bert(cfg)
    plan = g.partition(L.device_query(0))
    assert "pattern bert:" in plan.describe() and "not used" not in plan.describe().splitlines()[0]
    return plan, session(g, plan, og.bert_feed(gX, gpl, x, w), [gy]), gy


def _region(plan, s, name, dtype, shape):
    off, nb = plan.debug_region(name)
    t = s.ws[off:off + nb]
    return t.view(dtype).view(shape)


def _run_stages(s, b, e):
    os.environ["SOUFFLE_BERT_STAGES"] = f"{b},{e}"
    try:
        s.run()
        torch.cuda.synchronize()
    finally:
        del os.environ["SOUFFLE_BERT_STAGES"]


def test_qkv_stage_integer_bit_exact(record_err):
    S, H, nh = CFG["seq"], CFG["hidden"], CFG["heads"]
    w = synth.bert_weights(CFG, integer=True)
    x = synth.small_ints(77, (S, H))
    plan, s, _ = _session(CFG, w, x)
    _run_stages(s, 0, 2)                       # convert + QKV of layer 0
    L0 = w[0]
    q = x.astype(np.float64) @ L0["Wq"].astype(np.float64).T + L0["bq"]
    k = x.astype(np.float64) @ L0["Wk"].astype(np.float64).T + L0["bk"]
    v = x.astype(np.float64) @ L0["Wv"].astype(np.float64).T + L0["bv"]
    qk = _region(plan, s, "qk", torch.bfloat16, (2, nh, S, 64)).double().cpu().numpy()
    vt = _region(plan, s, "vt", torch.bfloat16, (nh, 64, S)).double().cpu().numpy()
    want_q = _bf16_rne(q).reshape(S, nh, 64).transpose(1, 0, 2)
    want_k = _bf16_rne(k).reshape(S, nh, 64).transpose(1, 0, 2)
    want_vt = _bf16_rne(v).reshape(S, nh, 64).transpose(1, 2, 0)
    mism = int((qk[0] != want_q).sum() + (qk[1] != want_k).sum() + (vt != want_vt).sum())
    record_err(mism, 0, what="mismatching Q/K/V^T elements")


def test_ffn2_stage_split_k_partials_integer_bit_exact(record_err):
    S, H, F = CFG["seq"], CFG["hidden"], CFG["ffn"]
    w = synth.bert_weights(CFG, integer=True)
    x = synth.small_ints(77, (S, H))
    plan, s, _ = _session(CFG, w, x)
    hin = synth.small_ints(78, (S, F))
    _region(plan, s, "h", torch.bfloat16, (S, F)).copy_(torch.from_numpy(hin).to(torch.bfloat16))
    part = _region(plan, s, "part_2", torch.float32, (-1, S, H))
    part.fill_(float("nan"))
    _run_stages(s, 5, 6)                       # FFN2 of layer 0 alone
    got = part.double().cpu().numpy()
    want = hin.astype(np.float64) @ w[0]["W2"].astype(np.float64).T
    ns = got.shape[0]
    kc = F // ns
    mism = 0
    for sp in range(ns):                       # every split-K partial is the exact K-range GEMM
        ref = hin[:, sp * kc:(sp + 1) * kc].astype(np.float64) @ w[0]["W2"][:, sp * kc:(sp + 1) * kc].astype(np.float64).T
        mism += int((got[sp] != ref).sum())
    mism += int((got.sum(0) != want).sum())
    record_err(mism, 0, what="mismatching FFN2 partial elements", nsplit=ns)


def test_ffn1_stage_gelu_integer_inputs(record_err):
    """FFN1 (+bias, erf-GELU, bf16): the pre-activation is an exact integer; the output must be the
    bf16 rounding of GELU of it, up to one bf16 ulp (fp32 erff vs fp64 erf at a rounding boundary)."""
    import math
    S, H, F = CFG["seq"], CFG["hidden"], CFG["ffn"]
    w = synth.bert_weights(CFG, integer=True)
    x = synth.small_ints(77, (S, H))
    plan, s, _ = _session(CFG, w, x)
    s.run()                                    # stage 0 of a full launch refreshes the packed bias vectors
    a = synth.small_ints(79, (S, H))
    _region(plan, s, "l1b", torch.bfloat16, (S, H)).copy_(torch.from_numpy(a).to(torch.bfloat16))
    _run_stages(s, 4, 5)
    got = _region(plan, s, "h", torch.bfloat16, (S, F)).double().cpu().numpy()
    pre = a.astype(np.float64) @ w[0]["W1"].astype(np.float64).T + w[0]["c1"]
    erf = np.vectorize(math.erf)
    want = _bf16_rne(0.5 * pre * (1.0 + erf(pre / math.sqrt(2.0))))
    # one bf16 ulp (2^-7 relative, upper bound) or 1e-6 absolute (GELU of a large negative
    # pre-activation is ~1e-23 in fp64 and exactly 0 with fp32 erff)
    bound = np.abs(want) * 2.0 ** -7 + 1e-6
    record_err(float(np.max(np.abs(got - want) / bound)), 1.0, what="max error in units of (1 bf16 ulp + 1e-6)")


def _ln_case(kind):
    """1 layer with Wo = W2 = 0 and bo = c2 = 0: y1 = x, so LN1 sees the input rows directly."""
    S, H = CFG["seq"], CFG["hidden"]
    w = synth.bert_weights(CFG)
    w[0]["Wo"] = np.zeros_like(w[0]["Wo"])
    w[0]["W2"] = np.zeros_like(w[0]["W2"])
    w[0]["bo"] = np.zeros_like(w[0]["bo"])
    w[0]["c2"] = np.zeros_like(w[0]["c2"])
    if kind == "constant":
        x = np.repeat((np.arange(S, dtype=np.float32) * 0.37 - 20.0)[:, None], H, axis=1).astype(np.float32)
        x[::7] = 1000.0
    else:
        x = (1000.0 + synth.normal(91, (S, H))).astype(np.float32)
    return w, x


@pytest.mark.parametrize("kind", ["constant", "offset"])
def test_layernorm_degenerate_rows(kind, record_err):
    """SURVEY §8(c) LayerNorm pins on the kernel: a constant row normalises to exactly beta (eps =
    1e-12 amplifies any error in the mean by 1e6), a row 1e3 + N(0,1) keeps its noise."""
    w, x = _ln_case(kind)
    spec, X, plist, y = og.bert(CFG)
    feed = og.bert_feed(X, plist, x, w)
    ref = te.evaluate(spec, feed)[y]
    if kind == "constant":
        l1 = [i for i, n in enumerate(spec["nodes"]) if n["op"] == "ew" and n["fn"] == "add"]
        vals = te.evaluate(spec, feed)
        assert any(np.array_equal(vals[i], np.broadcast_to(w[0]["be1"], vals[i].shape)) for i in l1)
    plan, s, gy = _session(CFG, w, x)
    s.run()
    out = s.result(gy)
    record_err(float(np.abs(out - ref).max()), 2e-2, kind=kind)


def test_bound_bias_updated_in_place_is_seen(record_err):
    """Constant vectors are refreshed from the bound pointers by every launch (no stale snapshot)."""
    cfg = dict(CFG)
    w = synth.bert_weights(cfg)
    x = synth.bert_input(cfg)
    g, gX, gpl, gy = M.bert(cfg)
    plan = g.partition(L.device_query(0))
    s = session(g, plan, og.bert_feed(gX, gpl, x, w), [gy])
    s.run()
    out0 = s.result(gy)
    w[0]["c1"] = (w[0]["c1"] + 0.5).astype(np.float32)
    w[0]["be2"] = (w[0]["be2"] - 0.25).astype(np.float32)
    s.inputs[gpl[0]["c1"]].copy_(torch.from_numpy(w[0]["c1"]))
    s.inputs[gpl[0]["be2"]].copy_(torch.from_numpy(w[0]["be2"]))
    s.run()
    out1 = s.result(gy)
    spec, X, plist, y = og.bert(cfg)
    emu = te.evaluate(spec, og.bert_feed(X, plist, x, w), bf16_operands=True)[y]
    assert np.abs(out1 - out0).max() > 0.1
    record_err(float(np.abs(out1 - emu).max()), 2e-2)


@pytest.mark.parametrize("kind", ["constant", "offset"])
def test_layernorm_degenerate_rows_generic_executor(kind, record_err):
    """The same LayerNorm pins on the generic fused executor (exec.cu, tiny fp32 BERT layer): the
    reduction stage's mean is shifted by the row's first element, so a constant row normalises to
    beta and an offset row keeps its noise (fp32 path tolerance: rel 1e-4 of max(|o|, rms))."""
    cfg = dict(synth.BERT_TINY)
    S, H = cfg["seq"], cfg["hidden"]
    w = synth.bert_weights(cfg)
    for k in ("Wo", "W2", "bo", "c2"):
        w[0][k] = np.zeros_like(w[0][k])
    if kind == "constant":
        x = np.repeat((np.arange(S, dtype=np.float32) * 0.37 - 5.0)[:, None], H, axis=1).astype(np.float32)
        x[::5] = 1000.0
    else:
        x = (1000.0 + synth.normal(92, (S, H))).astype(np.float32)
    spec, X, plist, y = og.bert(cfg)
    ref = te.evaluate(spec, og.bert_feed(X, plist, x, w))[y]
    g, gX, gpl, gy = M.bert(cfg)
    plan = g.partition(L.device_query(0))
    assert "pattern bert: not used" in plan.describe()
    s = session(g, plan, og.bert_feed(gX, gpl, x, w), [gy])
    s.run()
    out = s.result(gy)
    rms = np.sqrt(np.mean(ref ** 2))
    record_err(float(np.max(np.abs(out - ref) / np.maximum(np.abs(ref), rms))), 1e-4, kind=kind)
