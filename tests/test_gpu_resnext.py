"""GPU parity of the ResNeXt Bottleneck blocks (Table 2, ResNeXt-101 64 x 4d; SURVEY
§8(f) NEXT-3) on the pattern kernel and on the generic fused-subprogram executor against the fp64 oracle: fp32 TEs, max_i |g_i -
o_i| / max(|o_i|, rms(o)) <= 1e-4.  The grouped 3x3 convolution runs as 9 batched-matmul TEs over the
64 groups whose rolled + masked A operands are gathered through the index maps (stencil gathers)."""
import numpy as np
import pytest

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


def _case(cfg, flags=0):
    p = {**synth.resnext_params(cfg), **synth.resnext_masks(cfg)}
    x = synth.resnext_input(cfg)
    spec, on, ox, oy = og.resnext(cfg)
    ref = te.evaluate(spec, {on[k]: v for k, v in p.items()} | {ox: x})[oy]
    g, gn, gx, gy = M.resnext(cfg)
    plan = g.partition(L.device_query(0), flags)
    s = session(g, plan, {gn[k]: v for k, v in p.items()} | {gx: x}, [gy])
    s.run()
    s.run()   # repeated launches reuse the workspace
    return s.result(gy), ref, plan


@pytest.mark.parametrize("i", range(8), ids=[c["name"] for c in synth.RESNEXT_CONFIGS])
def test_resnext_block_pattern(i, record_err):
    """The ResNeXt pattern kernel (kernels/resnext.cu): one persistent launch, two grid barriers."""
    cfg = synth.RESNEXT_CONFIGS[i]
    out, ref, plan = _case(cfg)
    assert "pattern resnext:" in plan.describe() and plan.exec_info()["launches"] == 1
    record_err(rel_err(out, ref), 1e-4, block=cfg["name"], path="pattern")


@pytest.mark.parametrize("i", range(8), ids=[c["name"] for c in synth.RESNEXT_CONFIGS])
def test_resnext_block_generic(i, record_err):
    cfg = synth.RESNEXT_CONFIGS[i]
    out, ref, plan = _case(cfg, L.FLAG_NO_PATTERN)
    assert "pattern resnext: not used" in plan.describe()
    record_err(rel_err(out, ref), 1e-4, block=cfg["name"], launches=plan.exec_info()["launches"], path="generic")


@pytest.mark.parametrize("flags", [L.FLAG_UNFUSED, L.FLAG_NO_GLOBAL_SYNC])
def test_resnext_block_ablation_flags(flags, record_err):
    cfg = synth.RESNEXT_CONFIGS[3]
    out, ref, plan = _case(cfg, flags)
    record_err(rel_err(out, ref), 1e-4, block=cfg["name"], flags=flags)
