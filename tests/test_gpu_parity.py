"""GPU parity: the fused sm_100a path (through the C ABI) against the CPU fp64 oracle on the same
seeded inputs.  Tolerances (BASELINE.json north_star):
  * integer / GEMM-only stages with inputs in {-2..2}: bit-exact
  * fp32 paths: max_i |g_i - o_i| / max(|o_i|, rms(o)) <= 1e-4
  * bf16-operand paths: max abs <= 2e-2 on unit-scale activations (oracle with bf16 operand emulation)
"""
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


def rel_err(g, o):
    o = np.asarray(o, np.float64)
    g = np.asarray(g, np.float64)
    rms = np.sqrt(np.mean(o * o)) + 1e-30
    return float(np.max(np.abs(g - o) / np.maximum(np.abs(o), rms)))


def run(graph, feed, outs, flags=0):
    plan = graph.partition(L.device_query(0), flags)
    s = session(graph, plan, feed, outs)
    s.run()
    return [s.result(o) for o in outs], plan


def _gemm_graph(M_, N, K, relu_a, prec=L.BF16):
    g = L.Graph()
    X = g.placeholder((M_, K), L.F32, const=False)
    W = g.placeholder((N, K), L.BF16 if prec == L.BF16 else L.F32)
    A = g.ew("relu", X) if relu_a else X
    Y = g.matmul(A, W, True, prec)
    g.mark_output(Y)
    return g, X, W, Y


@pytest.mark.parametrize("M_,N,K,relu_a", [(128, 192, 256, False), (128, 192, 256, True), (128, 64, 64, True),
                                           (200, 128, 128, True), (128, 2304, 768, True)])
@pytest.mark.parametrize("flags", [0, L.FLAG_UNFUSED])
def test_tc_gemm_integer_bit_exact(M_, N, K, relu_a, flags):
    g, X, W, Y = _gemm_graph(M_, N, K, relu_a)
    x = synth.small_ints(11, (M_, K))
    w = synth.small_ints(12, (N, K), dtype="bf16")
    (y,), plan = run(g, {X: x, W: w}, [Y], flags)
    a = np.maximum(x, 0) if relu_a else x
    ref = a.astype(np.float64) @ w.astype(np.float64).T
    assert "GEMM_TC" in plan.describe()
    assert np.array_equal(y, ref), plan.describe()


def test_fig2_fp32_simt(record_err):
    spec, ids = og.fig2()
    ins = synth.spec_inputs(spec, 3)
    g, pids = M.fig2()
    (y,), _ = run(g, {i: v for i, v in ins.items()}, [pids["TE4"]])
    ref = te.evaluate(spec, ins)[ids["TE4"]]
    record_err(rel_err(y, ref), 1e-4)


@pytest.mark.parametrize("seed", range(8))
def test_random_programs_generic_path(seed, record_err):
    spec = synth.random_spec(seed, n_ops=20)
    ins = synth.spec_inputs(spec, seed)
    g = M.from_spec(spec)
    ref = te.evaluate(spec, ins)
    for flags in (0, L.FLAG_UNFUSED, L.FLAG_NO_GLOBAL_SYNC):
        outs, plan = run(g, ins, spec["outputs"], flags)
        for o, y in zip(spec["outputs"], outs):
            record_err(rel_err(y, ref[o]), 1e-4)


@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("cache", [None, "4096", "2048"])
def test_rowwise_programs_tensor_cache(seed, cache, monkeypatch, record_err):
    """§6.5 tensor reuse: row-wise reduction / elementwise programs whose stages hand
    each row block to the same CTA -- CTA-local dependencies without grid barriers, tensors kept in
    the shared-memory cache.  cache = SOUFFLE_CACHE_FLOATS: the default capacity, then capacities
    small enough that the LRU scan evicts tensors with readers still to come (spills to global) or
    cannot place them at all.  NO_PREFETCH turns reuse off; NO_GLOBAL_SYNC splits at the barriers."""
    if cache:
        monkeypatch.setenv("SOUFFLE_CACHE_FLOATS", cache)
    spec = synth.random_rowwise_spec(seed)
    ins = synth.spec_inputs(spec, seed)
    g = M.from_spec(spec)
    ref = te.evaluate(spec, ins)
    for flags in (0, L.FLAG_NO_PREFETCH, L.FLAG_NO_GLOBAL_SYNC):
        outs, plan = run(g, ins, spec["outputs"], flags)
        d = plan.describe()
        if flags & L.FLAG_NO_PREFETCH:
            assert "tensor cache" not in d
        for o, y in zip(spec["outputs"], outs):
            record_err(rel_err(y, ref[o]), 1e-4, flags=flags, cache=cache,
                       plan=[ln for ln in d.splitlines() if ln.startswith(("plan:", "tensor cache"))])


def test_tensor_cache_spills_are_exercised(monkeypatch):
    """The forced-capacity cases above really evict tensors with pending readers (host plan only)."""
    ev = 0
    for cache in ("4096", "2048"):
        monkeypatch.setenv("SOUFFLE_CACHE_FLOATS", cache)
        for seed in range(12):
            d = M.from_spec(synth.random_rowwise_spec(seed)).partition(L.device_query(0)).describe()
            ev += int(d.split("hit(s), ")[1].split(" LRU")[0])
    assert ev >= 3


@pytest.mark.parametrize("flags", [0, L.FLAG_UNFUSED, L.FLAG_NO_LN_REWRITE, L.FLAG_NO_VERTICAL])
def test_bert_tiny_fp32(flags, record_err):
    cfg = synth.BERT_TINY
    x = synth.bert_input(cfg)
    w = synth.bert_weights(cfg)
    spec, X, plist, y = og.bert(cfg)
    ref = te.evaluate(spec, og.bert_feed(X, plist, x, w))[y]
    g, gX, gpl, gy = M.bert(cfg)
    (out,), plan = run(g, og.bert_feed(gX, gpl, x, w), [gy], flags)
    record_err(rel_err(out, ref), 1e-4)


@pytest.mark.parametrize("layers,flags", [(1, 0), (1, L.FLAG_UNFUSED), (12, 0)])
def test_bert_base_bf16(layers, flags, record_err):
    cfg = dict(synth.BERT_BASE, layers=layers)
    x = synth.bert_input(cfg)
    w = synth.bert_weights(cfg)
    spec, X, plist, y = og.bert(cfg)
    feed = og.bert_feed(X, plist, x, w)
    emu = te.evaluate(spec, feed, bf16_operands=True)[y]
    g, gX, gpl, gy = M.bert(cfg)
    (out,), plan = run(g, og.bert_feed(gX, gpl, x, w), [gy], flags)
    err = float(np.abs(out - emu).max())
    record_err(err, 2e-2, vs="fp64 oracle, GEMM operands rounded to bf16", layers=layers, flags=flags)
    if layers == 1:
        exact = te.evaluate(spec, feed)[y]
        record_err(float(np.abs(out - exact).max()), 2e-2, vs="fp64 oracle", layers=layers, flags=flags)


@pytest.mark.parametrize("cfg,flags", [
    (synth.MMOE_CFG, 0),
    (synth.MMOE_CFG, L.FLAG_UNFUSED),
    (dict(synth.MMOE_CFG, batch=4, experts=5, tasks=3, expert_dim=24, tower_hidden=16, d_in=72, w_dtype="bf16"), 0),
])
def test_mmoe(cfg, flags, record_err):
    p = synth.mmoe_params(cfg)
    x = synth.mmoe_input(cfg)
    spec, names, outs = og.mmoe(cfg)
    feed = {names[k]: v for k, v in p.items()}
    feed[names["x"]] = x
    ref = te.evaluate(spec, feed)
    g, gn, gouts = M.mmoe(cfg)
    gfeed = {gn[k]: v for k, v in p.items()}
    gfeed[gn["x"]] = x
    res, plan = run(g, gfeed, gouts, flags)
    if flags == 0:
        assert "pattern mmoe:" in plan.describe() and "not used" not in plan.describe().splitlines()[2]
    for o, r in zip(outs, res):
        record_err(rel_err(r, ref[o]), 1e-4)


def test_mmoe_single_cta_kernel(monkeypatch, record_err):
    """The single-CTA MMoE kernel on the default configuration (the cluster kernel's shape), forced with
    SOUFFLE_MMOE_SINGLE=1; test_mmoe covers the cluster kernel (default) and the single kernel (batch 4)."""
    monkeypatch.setenv("SOUFFLE_MMOE_SINGLE", "1")
    cfg = synth.MMOE_CFG
    p = synth.mmoe_params(cfg)
    x = synth.mmoe_input(cfg)
    spec, names, outs = og.mmoe(cfg)
    feed = {names[k]: v for k, v in p.items()}
    feed[names["x"]] = x
    ref = te.evaluate(spec, feed)
    g, gn, gouts = M.mmoe(cfg)
    gfeed = {gn[k]: v for k, v in p.items()}
    gfeed[gn["x"]] = x
    res, plan = run(g, gfeed, gouts, 0)
    assert "in one CTA" in plan.describe()
    for o, r in zip(outs, res):
        record_err(rel_err(r, ref[o]), 1e-4)


def _lstm_case(cfg, flags=0, reps=1):
    x = synth.lstm_input(cfg)
    ps = synth.lstm_params(cfg)
    spec, names, top, hs, cs = og.lstm(cfg)

    def feed_for(nm):
        f = {nm["X"]: x}
        for n, p in enumerate(ps):
            f[nm[f"W{n}"]], f[nm[f"U{n}"]] = p["W"], p["U"]
            f[nm[f"bih{n}"]], f[nm[f"bhh{n}"]] = p["b_ih"], p["b_hh"]
            f[nm[f"h0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
            f[nm[f"c0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
        return f

    ref = te.evaluate(spec, feed_for(names))
    g, gn, gtop, ghs, gcs = M.lstm(cfg)
    outs = list(gtop) + list(ghs) + list(gcs)
    plan = g.partition(L.device_query(0), flags)
    s = session(g, plan, feed_for(gn), outs)
    for _ in range(reps):   # repeated launches reuse the workspace (run-generation tags)
        s.run()
    res = [s.result(o) for o in outs]
    T = len(gtop)
    got_top = np.concatenate(res[:T])
    want_top = np.concatenate([ref[t] for t in top])
    got_state = np.concatenate(res[T:])
    want_state = np.concatenate([ref[t] for t in list(hs) + list(cs)])
    return got_top, want_top, got_state, want_state, plan


@pytest.mark.parametrize("flags", [0, L.FLAG_UNFUSED])
def test_lstm_small_fp32(flags, record_err):
    cfg = dict(synth.LSTM_CFG, steps=5, layers=3, hidden=64, input=64, w_dtype="f32")
    gt, wt, gs, ws, plan = _lstm_case(cfg, flags)
    if flags == 0:
        assert "pattern lstm: 3 layers" in plan.describe()
    record_err(rel_err(gt, wt), 1e-4)
    record_err(rel_err(gs, ws), 1e-4)


def test_lstm_ragged_fp32(record_err):
    """3 CTAs per layer, input width != hidden width, odd step count."""
    cfg = dict(synth.LSTM_CFG, steps=7, layers=2, hidden=96, input=40, w_dtype="f32")
    gt, wt, gs, ws, plan = _lstm_case(cfg)
    assert "pattern lstm: 2 layers" in plan.describe()
    record_err(rel_err(gt, wt), 1e-4)
    record_err(rel_err(gs, ws), 1e-4)


@pytest.mark.parametrize("cfg_kw,force_smem", [
    (dict(steps=6, layers=3, hidden=64, input=64, w_dtype="f32"), True),     # shared-memory kernel, forced
    (dict(steps=5, layers=2, hidden=320, input=320, w_dtype="bf16"), False),  # K = 640 > 512: shared memory
    (dict(steps=5, layers=2, hidden=256, input=256, w_dtype="bf16"), True),   # full-width rows, forced
])
def test_lstm_shared_memory_kernel(cfg_kw, force_smem, monkeypatch, record_err):
    """The shared-memory LSTM kernel (rows too wide for the register-resident GEMV, or forced with
    SOUFFLE_LSTM_SMEM=1) stays parity-green next to the register-resident default."""
    if force_smem:
        monkeypatch.setenv("SOUFFLE_LSTM_SMEM", "1")
    cfg = dict(synth.LSTM_CFG, **cfg_kw)
    gt, wt, gs, ws, plan = _lstm_case(cfg, reps=2)
    d = plan.describe()
    assert "weights resident in shared memory" in d, d
    record_err(rel_err(gt, wt), 1e-4)
    record_err(rel_err(gs, ws), 1e-4)


def test_lstm_register_kernel_selected():
    """The default LSTM configuration runs the register-resident GEMV kernel."""
    _, _, _, _, plan = _lstm_case(dict(synth.LSTM_CFG, steps=3, layers=2), reps=1)
    assert "weights resident in registers" in plan.describe()


def test_lstm_full_config_bf16_weights(record_err):
    """BASELINE.json configs[2]: 10 stacked cells, hidden 256, 100 steps, batch 1 (persistent kernel,
    weights resident on chip).  bf16 weights are exact in the oracle; activations stay fp32."""
    gt, wt, gs, ws, plan = _lstm_case(synth.LSTM_CFG, reps=3)
    assert "pattern lstm: 10 layers x 100 steps" in plan.describe()
    record_err(rel_err(gt, wt), 1e-4)
    record_err(rel_err(gs, ws), 1e-4)


@pytest.mark.parametrize("seq,hidden,heads,ffn,layers", [
    (72, 768, 12, 3072, 2),     # ragged: 72 of the 128 rows of the M tile, masked softmax keys
    (8, 256, 4, 1024, 3),       # minimum multiple of 8 tokens, 4 heads, smaller FFN
    (128, 384, 6, 1536, 2),     # 6 heads: different tile counts in every stage
])
def test_bert_pattern_ragged_shapes(seq, hidden, heads, ffn, layers, record_err):
    """The persistent BERT kernel on shapes other than BERT-base (edge cases of its tile policy)."""
    cfg = dict(synth.BERT_BASE, seq=seq, hidden=hidden, heads=heads, ffn=ffn, layers=layers)
    x = synth.bert_input(cfg)
    w = synth.bert_weights(cfg)
    spec, X, plist, y = og.bert(cfg)
    emu = te.evaluate(spec, og.bert_feed(X, plist, x, w), bf16_operands=True)[y]
    g, gX, gpl, gy = M.bert(cfg)
    (out,), plan = run(g, og.bert_feed(gX, gpl, x, w), [gy])
    assert "pattern bert:" in plan.describe() and "not used" not in plan.describe().splitlines()[0]
    err = float(np.abs(out - emu).max())
    record_err(err, 2e-2)


def test_bert_seq_not_multiple_of_8_runs_generic(record_err):
    """S = 20 is outside the pattern kernel (V^T rows are TMA-loaded in 8s): the generic fused
    executor runs it, still matching the oracle."""
    cfg = dict(synth.BERT_BASE, seq=20, hidden=128, heads=2, ffn=512, layers=1)
    x = synth.bert_input(cfg)
    w = synth.bert_weights(cfg)
    spec, X, plist, y = og.bert(cfg)
    emu = te.evaluate(spec, og.bert_feed(X, plist, x, w), bf16_operands=True)[y]
    g, gX, gpl, gy = M.bert(cfg)
    (out,), plan = run(g, og.bert_feed(gX, gpl, x, w), [gy])
    assert "not used" in plan.describe().splitlines()[0]
    record_err(float(np.abs(out - emu).max()), 2e-2)


def test_bert_pattern_repeated_launches_reuse_workspace(record_err):
    """Three back-to-back launches on one workspace: the barrier counters are reset by the last CTA
    of each launch, so every launch must reproduce the oracle (and the same bits up to atomics-free
    determinism: the BERT kernel has no atomics on the data path)."""
    cfg = dict(synth.BERT_BASE, layers=2)
    x = synth.bert_input(cfg)
    w = synth.bert_weights(cfg)
    spec, X, plist, y = og.bert(cfg)
    emu = te.evaluate(spec, og.bert_feed(X, plist, x, w), bf16_operands=True)[y]
    g, gX, gpl, gy = M.bert(cfg)
    plan = g.partition(L.device_query(0))
    s = session(g, plan, og.bert_feed(gX, gpl, x, w), [gy])
    outs = []
    for _ in range(3):
        s.run()
        outs.append(s.result(gy))
    for o in outs:
        record_err(float(np.abs(o - emu).max()), 2e-2)
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[1], outs[2])


@pytest.mark.parametrize("flags", [L.FLAG_NO_PATTERN, L.FLAG_NO_PATTERN | L.FLAG_NO_GLOBAL_SYNC])
def test_lstm_generic_fused_executor(flags, record_err):
    """The generic fused executor on a stacked LSTM with hidden 256: horizontally fused GEMV groups of
    several members (warp-per-output skinny-GEMM path, member switches inside a CTA's task loop)."""
    cfg = dict(synth.LSTM_CFG, steps=12, layers=4, hidden=256, input=256, w_dtype="f32")
    gt, wt, gs, ws, plan = _lstm_case(cfg, flags, reps=2)
    assert "GEMM_SIMT" in plan.describe()
    record_err(rel_err(gt, wt), 1e-4)
    record_err(rel_err(gs, ws), 1e-4)


@pytest.mark.parametrize("flags", [L.FLAG_NO_PATTERN, L.FLAG_NO_PATTERN | L.FLAG_NO_VERTICAL | L.FLAG_NO_GLOBAL_SYNC])
def test_bert_base_generic_fused_executor(flags, record_err):
    """BERT-base (2 layers) on the generic fused executor (the Table 4 V1 / V3 rungs)."""
    cfg = dict(synth.BERT_BASE, layers=2)
    x = synth.bert_input(cfg)
    w = synth.bert_weights(cfg)
    spec, X, plist, y = og.bert(cfg)
    emu = te.evaluate(spec, og.bert_feed(X, plist, x, w), bf16_operands=True)[y]
    g, gX, gpl, gy = M.bert(cfg)
    (out,), plan = run(g, og.bert_feed(gX, gpl, x, w), [gy], flags)
    assert "not used" in plan.describe().splitlines()[0]
    record_err(float(np.abs(out - emu).max()), 2e-2)
