"""Oracle pins for the Swin-Transformer TE program (Table 2).

The oracle's Swin graph (oracle/graphs.swin) is pinned against torchvision's SwinTransformer run in
fp64 with the same weights copied in -- an implementation written independently of ours (its own
roll, window partition, mask construction and relative-position gather).  The roll TE is pinned by
its element-by-element definition (brute mode) on a small tensor."""
import numpy as np
import pytest
import torch

import synth
import synth.swin as S
from oracle import graphs as G
from oracle import te


def _torchvision_model(cfg, P):
    from torchvision.models.swin_transformer import SwinTransformer
    m = SwinTransformer(patch_size=[cfg["patch"]] * 2, embed_dim=cfg["embed"], depths=list(cfg["depths"]),
                        num_heads=list(cfg["heads"]), window_size=[cfg["window"]] * 2, mlp_ratio=cfg["mlp_ratio"],
                        stochastic_depth_prob=0.0, num_classes=cfg["classes"]).double().eval()
    T = lambda a: torch.from_numpy(np.asarray(a, dtype=np.float64))
    f = m.features
    C, p = cfg["embed"], cfg["patch"]
    with torch.no_grad():
        f[0][0].weight.copy_(T(P["Wpe"]).reshape(C, 3, p, p))
        f[0][0].bias.copy_(T(P["bpe"]))
        f[0][2].weight.copy_(T(P["gpe"]))
        f[0][2].bias.copy_(T(P["bepe"]))
        gb = 0
        for i, depth in enumerate(cfg["depths"]):
            stage = f[1 + 2 * i]
            for j in range(depth):
                blk, bp = stage[j], P["blocks"][gb]
                blk.norm1.weight.copy_(T(bp["g1"]))
                blk.norm1.bias.copy_(T(bp["be1"]))
                blk.attn.qkv.weight.copy_(T(bp["Wqkv"]))
                blk.attn.qkv.bias.copy_(T(bp["bqkv"]))
                blk.attn.relative_position_bias_table.copy_(T(bp["table"]))
                blk.attn.proj.weight.copy_(T(bp["Wproj"]))
                blk.attn.proj.bias.copy_(T(bp["bproj"]))
                blk.norm2.weight.copy_(T(bp["g2"]))
                blk.norm2.bias.copy_(T(bp["be2"]))
                blk.mlp[0].weight.copy_(T(bp["W1"]))
                blk.mlp[0].bias.copy_(T(bp["b1"]))
                blk.mlp[3].weight.copy_(T(bp["W2"]))
                blk.mlp[3].bias.copy_(T(bp["b2"]))
                gb += 1
            if i < len(cfg["depths"]) - 1:
                mg, mp = f[2 + 2 * i], P["merges"][i]
                mg.norm.weight.copy_(T(mp["g"]))
                mg.norm.bias.copy_(T(mp["be"]))
                mg.reduction.weight.copy_(T(mp["W"]))
        m.norm.weight.copy_(T(P["gn"]))
        m.norm.bias.copy_(T(P["ben"]))
        m.head.weight.copy_(T(P["Wh"]))
        m.head.bias.copy_(T(P["bh"]))
    return m


def _oracle_logits(cfg, P, img):
    spec, names, x, y = G.swin(cfg)
    fv = S.swin_feed_values(cfg, P)
    assert set(fv) == set(names)
    inp = {names[k]: v for k, v in fv.items()}
    inp[x] = img
    return te.evaluate(spec, inp)[y]


@pytest.mark.parametrize("batch", [1, 2])
def test_swin_tiny_matches_torchvision_fp64(batch):
    cfg = dict(S.SWIN_TINY, batch=batch)
    P = S.swin_params(cfg)
    img = S.swin_input(cfg)
    ours = _oracle_logits(cfg, P, img)
    with torch.no_grad():
        ref = _torchvision_model(cfg, P)(torch.from_numpy(img.astype(np.float64))).numpy()
    assert ours.shape == ref.shape
    np.testing.assert_allclose(ours, ref, rtol=1e-10, atol=1e-10)


def test_swin_three_stages_shift_and_no_shift_match_torchvision():
    """image 112 -> 28, 14, 7: shifted stages 1-2 (4x4 and 2x2 windows) and an unshifted stage."""
    cfg = dict(S.SWIN_TINY, image=112, depths=(2, 2, 2), heads=(1, 2, 4), embed=16)
    P = S.swin_params(cfg)
    img = S.swin_input(cfg)
    ours = _oracle_logits(cfg, P, img)
    with torch.no_grad():
        ref = _torchvision_model(cfg, P)(torch.from_numpy(img.astype(np.float64))).numpy()
    np.testing.assert_allclose(ours, ref, rtol=1e-10, atol=1e-10)


def test_swin_mask_and_bias_change_the_result():
    """The bias and mask inputs are live: perturbing them changes the oracle's logits."""
    cfg = S.SWIN_TINY
    P = S.swin_params(cfg)
    img = S.swin_input(cfg)
    spec, names, x, y = G.swin(cfg)
    fv = S.swin_feed_values(cfg, P)
    base = {names[k]: v for k, v in fv.items()}
    base[x] = img
    y0 = te.evaluate(spec, base)[y]
    for key in ("b1.mask", "b0.bias"):
        alt = dict(base)
        alt[names[key]] = np.zeros_like(fv[key])
        assert np.abs(te.evaluate(spec, alt)[y] - y0).max() > 1e-3, key


def test_roll_brute_definition():
    spec = {"nodes": [dict(op="placeholder", shape=[3, 5, 4], dtype="f32", const=0),
                      {"op": "roll", "in": 0, "shifts": [1, -2, 0]}], "outputs": [1]}
    x = synth.normal(7, (3, 5, 4))
    v = te.evaluate(spec, {0: x})[1]
    b = te.evaluate(spec, {0: x}, brute=True)[1]
    np.testing.assert_array_equal(v, b)
    # out[i, j, k] = x[(i - 1) % 3, (j + 2) % 5, k]
    assert v[0, 0, 1] == np.float64(x[2, 2, 1])
    assert v[1, 4, 3] == np.float64(x[0, 1, 3])


def test_shift_mask_regions():
    """Mask: 0 inside one region, -100 across regions; the un-wrapped top-left windows are all 0."""
    m = S.shift_mask(14, 7, 3)
    assert m.shape == (4, 1, 49, 49)
    assert np.all(m[0] == 0)
    assert set(np.unique(m)) == {0.0, -100.0}
    assert np.all(m[3, 0].diagonal() == 0)
