"""Oracle pins for the EfficientNet MBConv blocks M0-M9 (Fig. 5 / 6, L1511-1564: "the
sub-module is the building block of EfficientNet"): the oracle's TE program -- 1x1 convolutions as
matmuls, the depthwise convolution as rolled and border-masked taps, SE, BatchNorm in inference form
-- against torchvision's MBConv (real zero-padded grouped Conv2d) in fp64 with the same weights; the
library builds the identical node sequence."""
import numpy as np
import pytest
import torch

import synth
from oracle import graphs as og
from oracle import te


def _torch_mbconv(cfg, p):
    from functools import partial

    from torchvision.models.efficientnet import MBConv, MBConvConfig
    d = synth.mbconv_dims(cfg)
    cin, cout, exp, S, k = cfg["cin"], cfg["cout"], d["exp"], d["squeeze"], cfg["k"]
    eps = 1e-5
    m = MBConv(MBConvConfig(cfg["expand"], k, cfg["stride"], cin, cout, 1), 0.0,
               partial(torch.nn.BatchNorm2d, eps=eps)).double().eval()
    blk = list(m.block)

    def set_bn(bn, s, b):   # running stats (0, 1): bn(x) = x * weight / sqrt(1 + eps) + bias
        bn.running_mean.zero_()
        bn.running_var.fill_(1.0)
        bn.weight.copy_(torch.from_numpy(s.astype(np.float64)) * np.sqrt(1.0 + eps))
        bn.bias.copy_(torch.from_numpy(b.astype(np.float64)))

    def t64(a):
        return torch.from_numpy(a.astype(np.float64))
    with torch.no_grad():
        i = 0
        if cfg["expand"] != 1:
            blk[0][0].weight.copy_(t64(p["We"]).view(exp, cin, 1, 1))
            set_bn(blk[0][1], p["se"], p["be"])
            i = 1
        dw = np.stack([p[f"w{t}"] for t in range(k * k)], 1).reshape(exp, 1, k, k)
        blk[i][0].weight.copy_(t64(dw))
        set_bn(blk[i][1], p["sd"], p["bd"])
        se = blk[i + 1]
        se.fc1.weight.copy_(t64(p["W1"]).view(S, exp, 1, 1))
        se.fc1.bias.copy_(t64(p["b1"]))
        se.fc2.weight.copy_(t64(p["W2"]).view(exp, S, 1, 1))
        se.fc2.bias.copy_(t64(p["b2"]))
        blk[i + 2][0].weight.copy_(t64(p["Wp"]).view(cout, exp, 1, 1))
        set_bn(blk[i + 2][1], p["sp"], p["bp"])
    return m


@pytest.mark.parametrize("cfg", synth.MBCONV_CONFIGS, ids=[c["name"] for c in synth.MBCONV_CONFIGS])
def test_mbconv_matches_torchvision(cfg):
    H = cfg["hw"]
    x = synth.mbconv_input(cfg)
    p = synth.mbconv_params(cfg)
    spec, names, X, Y = og.mbconv(cfg)
    feed = {names[k]: v for k, v in {**p, **synth.mbconv_masks(cfg)}.items()}
    feed[X] = x
    got = te.evaluate(spec, feed)[Y]
    m = _torch_mbconv(cfg, p)
    with torch.no_grad():
        img = torch.from_numpy(x.astype(np.float64)).view(1, H, H, cfg["cin"]).permute(0, 3, 1, 2)
        ref = m(img).permute(0, 2, 3, 1).reshape(-1, cfg["cout"]).numpy()
    assert got.shape == ref.shape
    assert np.max(np.abs(got - ref)) <= 1e-10 * max(1.0, np.max(np.abs(ref)))


def test_mbconv_library_graph_matches_oracle():
    from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L
    from paper_conf_asplos_xiazswwyfc24_b200 import models as M
    opmap = {"placeholder": 0, "matmul": 1, "ew": 2, "reduce": 3, "reshape": 4, "permute": 5, "slice": 6, "roll": 7}
    for cfg in (synth.MBCONV_CONFIGS[0], synth.MBCONV_CONFIGS[3]):
        spec, names, X, Y = og.mbconv(cfg)
        g, gnames, gx, gy = M.mbconv(cfg)
        assert g.num_nodes() == len(spec["nodes"]) and gnames == names and (gx, gy) == (X, Y)
        shapes = te.infer_shapes(spec)
        for i, nd in enumerate(spec["nodes"]):
            op, shp, _ = g.node(i)
            assert op == opmap[nd["op"]] and shp == shapes[i], i
        assert g.partition(L.device_b200()).num_subprograms() >= 1


def test_mbconv_pattern_matcher():
    """Every module M0-M9 is recognised by the MBConv pattern lowering (one persistent launch); the
    ablation flags keep the generic executor; a program that is not exactly the block is refused."""
    from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L
    from paper_conf_asplos_xiazswwyfc24_b200 import models as M
    for cfg in synth.MBCONV_CONFIGS:
        g = M.mbconv(cfg)[0]
        d = g.partition(L.device_b200()).describe()
        assert "pattern mbconv: " in d and "pattern mbconv: not used" not in d, cfg["name"]
        assert g.partition(L.device_b200()).exec_info()["launches"] == 1
        assert "pattern mbconv: not used" in g.partition(L.device_b200(), L.FLAG_NO_PATTERN).describe()
    g = M.se_module(synth.SE_CONFIGS[0])[0]
    assert "pattern mbconv: not used" in g.partition(L.device_b200()).describe()
