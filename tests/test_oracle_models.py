"""Pins for the oracle's model-level definitions: the TE programs (oracle/graphs.py) interpreted by
oracle/te.py must equal (a) the direct formulas (oracle/models.py) and (b) torch.nn reference
modules in fp64 with copied weights (independent library implementations)."""
import json
import math
import os

import numpy as np
import pytest
import torch

import synth
from oracle import graphs, models, te

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _torch_encoder(cfg, p):
    H, nh, F = cfg["hidden"], cfg["heads"], cfg["ffn"]
    layer = torch.nn.TransformerEncoderLayer(H, nh, F, dropout=0.0, activation="gelu",
                                             layer_norm_eps=cfg["eps"], batch_first=True).double()
    t = lambda a: torch.tensor(np.asarray(a, dtype=np.float64))
    with torch.no_grad():
        layer.self_attn.in_proj_weight.copy_(torch.cat([t(p["Wq"]), t(p["Wk"]), t(p["Wv"])]))
        layer.self_attn.in_proj_bias.copy_(torch.cat([t(p["bq"]), t(p["bk"]), t(p["bv"])]))
        layer.self_attn.out_proj.weight.copy_(t(p["Wo"]))
        layer.self_attn.out_proj.bias.copy_(t(p["bo"]))
        layer.linear1.weight.copy_(t(p["W1"]))
        layer.linear1.bias.copy_(t(p["c1"]))
        layer.linear2.weight.copy_(t(p["W2"]))
        layer.linear2.bias.copy_(t(p["c2"]))
        layer.norm1.weight.copy_(t(p["g1"]))
        layer.norm1.bias.copy_(t(p["be1"]))
        layer.norm2.weight.copy_(t(p["g2"]))
        layer.norm2.bias.copy_(t(p["be2"]))
    layer.eval()
    return layer


@pytest.mark.parametrize("cfg", [synth.BERT_TINY, dict(synth.BERT_BASE, layers=1)])
def test_bert_layer_vs_torch_encoder_layer(cfg):
    x = synth.bert_input(cfg)
    p = synth.bert_layer_weights(cfg, 0)
    spec, X, plist, y = graphs.bert(cfg, layers=1)
    vals = te.evaluate(spec, graphs.bert_feed(X, plist, x, [p]))
    direct = models.bert_layer(x, p, cfg["heads"], cfg["eps"])
    np.testing.assert_allclose(vals[y], direct, atol=1e-11, rtol=0)
    with torch.no_grad():
        ref = _torch_encoder(cfg, p)(torch.tensor(x, dtype=torch.float64)[None])[0].numpy()
    np.testing.assert_allclose(vals[y], ref, atol=1e-10, rtol=0)


def test_bert_bf16_emulation_close_to_fp64():
    """The bf16-operand emulation differs from the fp64 definition by bf16 operand rounding only."""
    cfg = dict(synth.BERT_BASE, layers=1)
    x = synth.bert_input(cfg)
    p = synth.bert_layer_weights(cfg, 0)
    spec, X, plist, y = graphs.bert(cfg, layers=1)
    feed = graphs.bert_feed(X, plist, x, [p])
    a = te.evaluate(spec, feed)[y]
    b = te.evaluate(spec, feed, bf16_operands=True)[y]
    d = models.bert_layer(x, p, cfg["heads"], cfg["eps"], bf16_operands=True)
    np.testing.assert_allclose(b, d, atol=1e-10)
    err = np.abs(a - b).max()
    assert 1e-4 < err < 2e-2, err


def test_lstm_vs_torch_lstm():
    cfg = dict(synth.LSTM_CFG, steps=6, layers=3, hidden=16, input=16)
    x = synth.lstm_input(cfg)
    ps = synth.lstm_params(cfg)
    spec, names, top, hs, cs = graphs.lstm(cfg)
    feed = {names["X"]: x}
    for n, p in enumerate(ps):
        feed[names[f"W{n}"]] = p["W"]
        feed[names[f"U{n}"]] = p["U"]
        feed[names[f"bih{n}"]] = p["b_ih"]
        feed[names[f"bhh{n}"]] = p["b_hh"]
        feed[names[f"h0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
        feed[names[f"c0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
    vals = te.evaluate(spec, feed)
    got_top = np.concatenate([vals[t] for t in top], axis=0)
    d_top, d_h, d_c = models.lstm(x, ps, cfg["hidden"])
    np.testing.assert_allclose(got_top, d_top, atol=1e-14)
    m = torch.nn.LSTM(cfg["input"], cfg["hidden"], cfg["layers"]).double()
    with torch.no_grad():
        for n, p in enumerate(ps):
            getattr(m, f"weight_ih_l{n}").copy_(torch.tensor(p["W"].astype(np.float64)))
            getattr(m, f"weight_hh_l{n}").copy_(torch.tensor(p["U"].astype(np.float64)))
            getattr(m, f"bias_ih_l{n}").copy_(torch.tensor(p["b_ih"].astype(np.float64)))
            getattr(m, f"bias_hh_l{n}").copy_(torch.tensor(p["b_hh"].astype(np.float64)))
        out, (hn, cn) = m(torch.tensor(x.astype(np.float64))[:, None, :])
    np.testing.assert_allclose(got_top, out[:, 0].numpy(), atol=1e-13)
    for n in range(cfg["layers"]):
        np.testing.assert_allclose(vals[hs[n]][0], hn[n, 0].numpy(), atol=1e-13)
        np.testing.assert_allclose(vals[cs[n]][0], cn[n, 0].numpy(), atol=1e-13)


def test_lstm_hand_stepped_two_timesteps():
    g = json.load(open(os.path.join(GOLD, "lstm_2step.json")))
    cfg = dict(synth.LSTM_CFG, steps=2, layers=1, hidden=1, input=1)
    spec, names, top, hs, cs = graphs.lstm(cfg)
    W = np.array([[math.log(v)] for v in g["W_ih_log_args"]])
    feed = {names["X"]: np.array(g["x"])[:, None], names["W0"]: W, names["U0"]: np.zeros((4, 1)),
            names["bih0"]: np.zeros(4), names["bhh0"]: np.zeros(4), names["h0_0"]: np.zeros((1, 1)),
            names["c0_0"]: np.zeros((1, 1))}
    vals = te.evaluate(spec, feed)
    # c values are exact rationals: 9/20 then 9/40
    assert abs(vals[top[0]][0, 0] - 0.75 * math.tanh(9 / 20)) < 1e-15
    assert abs(vals[top[1]][0, 0] - 0.5 * math.tanh(9 / 40)) < 1e-15
    assert abs(vals[cs[0]][0, 0] - 9 / 40) < 1e-15


def test_mmoe_graph_vs_formula_and_gate_rows_sum_to_one():
    cfg = synth.MMOE_CFG
    p = synth.mmoe_params(cfg)
    x = synth.mmoe_input(cfg)
    spec, names, outs = graphs.mmoe(cfg)
    feed = {names[k]: v for k, v in p.items()}
    feed[names["x"]] = x
    vals = te.evaluate(spec, feed)
    ys = models.mmoe(x, p, cfg)
    for o, y in zip(outs, ys):
        np.testing.assert_allclose(vals[o], y, atol=1e-13)
    # gate softmax outputs (the 'div' TEs) sum to 1
    divs = [i for i, n in enumerate(spec["nodes"]) if n["op"] == "ew" and n["fn"] == "div"]
    assert len(divs) == cfg["tasks"]
    for d in divs:
        np.testing.assert_allclose(vals[d].sum(axis=1), 1.0, atol=1e-14)


def test_fig2_graph_vs_formula():
    spec, ids = graphs.fig2()
    ins = synth.spec_inputs(spec, 3)
    vals = te.evaluate(spec, ins)
    np.testing.assert_allclose(vals[ids["TE4"]], models.fig2(ins[0], ins[1], ins[4], ins[7]), rtol=1e-13)
