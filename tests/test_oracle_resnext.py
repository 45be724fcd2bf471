"""Oracle pins for the ResNeXt Bottleneck blocks R0-R7 (Table 2: ResNeXt-101, 64
groups x 4d): the oracle's TE program -- 1x1 convolutions as matmuls, the grouped 3x3 convolution as
rolled + border-masked taps, each ONE batched matmul over the 64 groups, BatchNorm in inference form --
against torchvision's Bottleneck (a real zero-padded Conv2d with groups=64, strided) in fp64 with the
same weights; the library builds the identical node sequence."""
import numpy as np
import pytest
import torch

import synth
from oracle import graphs as og
from oracle import te


def _torch_block(cfg, p):
    from torchvision.models.resnet import Bottleneck, conv1x1
    cin, w, cout, G, s = cfg["cin"], cfg["width"], cfg["cout"], cfg["groups"], cfg["stride"]
    cg, eps = w // G, 1e-5
    down = None
    if synth.resnext_projection(cfg):
        down = torch.nn.Sequential(conv1x1(cin, cout, s), torch.nn.BatchNorm2d(cout, eps=eps))
    m = Bottleneck(cin, w // 4, s, down, groups=G, base_width=4).double().eval()
    assert m.conv2.weight.shape == (w, cg, 3, 3) and m.conv3.weight.shape == (cout, w, 1, 1)

    def set_bn(bn, sc, b):   # running stats (0, 1): bn(x) = x * weight / sqrt(1 + eps) + bias
        bn.running_mean.zero_()
        bn.running_var.fill_(1.0)
        bn.weight.copy_(torch.from_numpy(sc.astype(np.float64)) * np.sqrt(1.0 + eps))
        bn.bias.copy_(torch.from_numpy(b.astype(np.float64)))

    def t64(a):
        return torch.from_numpy(np.ascontiguousarray(a).astype(np.float64))
    with torch.no_grad():
        m.conv1.weight.copy_(t64(p["W1"]).view(w, cin, 1, 1))
        set_bn(m.bn1, p["s1"], p["b1"])
        # weight[g * cg + o, i_in, i, j] = W2_{3 i + j}[g, o, i_in]
        k = np.stack([p[f"W2_{t}"] for t in range(9)], -1).reshape(G, cg, cg, 3, 3).reshape(w, cg, 3, 3)
        m.conv2.weight.copy_(t64(k))
        set_bn(m.bn2, p["s2"], p["b2"])
        m.conv3.weight.copy_(t64(p["W3"]).view(cout, w, 1, 1))
        set_bn(m.bn3, p["s3"], p["b3"])
        if down is not None:
            down[0].weight.copy_(t64(p["Wd"]).view(cout, cin, 1, 1))
            set_bn(down[1], p["sd"], p["bd"])
    return m


@pytest.mark.parametrize("cfg", synth.RESNEXT_CONFIGS[:6], ids=[c["name"] for c in synth.RESNEXT_CONFIGS[:6]])
def test_resnext_block_matches_torchvision(cfg):
    """R0-R5 (R6 / R7 are the same code path at 2048 channels; their fp64 evaluation takes minutes)."""
    H, s = cfg["hw"], cfg["stride"]
    x = synth.resnext_input(cfg)
    p = synth.resnext_params(cfg)
    spec, names, X, Y = og.resnext(cfg)
    feed = {names[k]: v for k, v in {**p, **synth.resnext_masks(cfg)}.items()}
    feed[X] = x
    y = te.evaluate(spec, feed)[Y]
    m = _torch_block(cfg, p)
    xt = torch.from_numpy(x.astype(np.float64)).view(H, H, cfg["cin"]).permute(2, 0, 1).unsqueeze(0)
    with torch.no_grad():
        ref = m(xt)[0].permute(1, 2, 0).reshape((H // s) ** 2, cfg["cout"]).numpy()
    assert y.shape == ref.shape
    assert np.max(np.abs(y - ref)) <= 1e-9 * max(1.0, np.max(np.abs(ref)))


def test_resnext_grouped_taps_are_batched_matmuls():
    """Every tap of the grouped convolution is ONE batched matmul TE over the 64 groups (the
    horizontally transformed form of the 64 per-group convolutions, §6.1)."""
    cfg = synth.RESNEXT_CONFIGS[1]
    spec, names, X, Y = og.resnext(cfg)
    nodes = spec["nodes"]
    mms = [n for n in nodes if n["op"] == "matmul"]
    batched = [n for n in mms if nodes[n["b"]]["shape"] == [64, 4, 4]]
    assert len(batched) == 9 and all(nodes[n["a"]]["op"] == "permute" for n in batched)
    assert len(mms) == 9 + 2   # + the two 1x1 convolutions (R1: identity shortcut)
