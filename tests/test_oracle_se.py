"""Oracle pins for the EfficientNet squeeze-and-excitation sub-module M0-M9 (Fig. 5 / 6,
L1511-1564): the oracle's TE program against torchvision's SqueezeExcitation (AdaptiveAvgPool2d,
1x1 Conv2d fc1 + SiLU, 1x1 Conv2d fc2 + Sigmoid, channel scale) run in fp64 with the same weights
on the NCHW image of the same values; the library builds the identical TE program and analyses it
bit-exactly like the oracle."""
import numpy as np
import pytest
import torch

import synth
from oracle import analysis as an
from oracle import graphs as og
from oracle import te


@pytest.mark.parametrize("cfg", synth.SE_CONFIGS, ids=[c["name"] for c in synth.SE_CONFIGS])
def test_se_module_matches_torchvision(cfg):
    from torchvision.ops.misc import SqueezeExcitation
    H, C, S = cfg["hw"], cfg["channels"], cfg["squeeze"]
    x = synth.se_input(cfg)
    p = synth.se_params(cfg)
    spec, names, X, Y = og.se_module(cfg)
    feed = {names[k]: v for k, v in p.items()}
    feed[X] = x
    got = te.evaluate(spec, feed)[Y]
    m = SqueezeExcitation(C, S, activation=torch.nn.SiLU).double()   # efficientnet_b0 uses SiLU
    with torch.no_grad():
        m.fc1.weight.copy_(torch.from_numpy(p["W1"].astype(np.float64)).view(S, C, 1, 1))
        m.fc1.bias.copy_(torch.from_numpy(p["b1"].astype(np.float64)))
        m.fc2.weight.copy_(torch.from_numpy(p["W2"].astype(np.float64)).view(C, S, 1, 1))
        m.fc2.bias.copy_(torch.from_numpy(p["b2"].astype(np.float64)))
        img = torch.from_numpy(x.astype(np.float64)).view(1, H, H, C).permute(0, 3, 1, 2)
        ref = m(img).permute(0, 2, 3, 1).reshape(H * H, C).numpy()
    assert np.max(np.abs(got - ref)) <= 1e-12


def test_se_module_structure_and_library_graph():
    """Classification: the pool and both GEMVs are memory-intensive (ratio < 3), so the whole module is
    one subprogram (one kernel, Fig. 5(c)); the library builds the same node sequence."""
    from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L
    from paper_conf_asplos_xiazswwyfc24_b200 import models as M
    cfg = synth.SE_CONFIGS[9]
    spec, names, X, Y = og.se_module(cfg)
    info = an.classify(spec)
    assert not any(i["ci"] for i in info)
    g, gnames, gx, gy = M.se_module(cfg)
    assert g.num_nodes() == len(spec["nodes"]) and gnames == names and (gx, gy) == (X, Y)
    shapes = te.infer_shapes(spec)
    for i in range(len(spec["nodes"])):
        assert g.node(i)[1] == shapes[i]
    plan = g.partition(L.device_b200())
    assert plan.num_subprograms() == 1
    assert plan.assignment() == an.partition(spec, {i: (1, 0, 0, 0) for i in range(len(spec["nodes"]))},
                                             dict(rule=0, capacity_C=0, num_sms=148, smem_per_sm=233472,
                                                  smem_reserved_per_block=1024, regs_per_sm=65536,
                                                  max_threads_per_sm=2048, max_blocks_per_sm=32))
