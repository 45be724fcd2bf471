"""GPU parity of the EfficientNet MBConv blocks M0-M9 (Fig. 5 / 6, L1511-1564) against the
fp64 oracle: the pattern kernel (kernels/mbconv.cu: one persistent launch, Fig. 5(c)), and the
generic TE-program executor, where the depthwise convolution runs as the rolled / masked taps of the
TE program (composed quasi-affine index maps, §6.2), the 1x1 convolutions as GEMM stages with
BatchNorm + SiLU epilogues, SE as reduction + GEMV stages -- unfused (a), fused kernels launched
separately (b), one launch per subprogram (c).  fp32: max_i |g - o| / max(|o|, rms(o)) <= 1e-4."""
import numpy as np
import pytest

import synth
from oracle import graphs as og
from oracle import te
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L
from paper_conf_asplos_xiazswwyfc24_b200 import models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session

pytestmark = pytest.mark.gpu

VARIANTS = {"a_unfused": L.FLAG_UNFUSED, "b_fused": L.FLAG_NO_GLOBAL_SYNC,
            "c_generic_global_sync": L.FLAG_NO_PATTERN | L.FLAG_NO_PREFETCH}


def rel_err(g, o):
    rms = np.sqrt(np.mean(o * o)) + 1e-30
    return float(np.max(np.abs(g - o) / np.maximum(np.abs(o), rms)))


def _case(cfg):
    x = synth.mbconv_input(cfg)
    p = {**synth.mbconv_params(cfg), **synth.mbconv_masks(cfg)}
    spec, names, X, Y = og.mbconv(cfg)
    ref = te.evaluate(spec, {names[k]: v for k, v in p.items()} | {X: x})[Y]
    g, gnames, gx, gy = M.mbconv(cfg)
    return g, {gnames[k]: v for k, v in p.items()} | {gx: x}, gy, ref


@pytest.mark.parametrize("flags", [0, L.FLAG_NO_PREFETCH], ids=["reuse", "global_sync"])
@pytest.mark.parametrize("cfg", synth.MBCONV_CONFIGS, ids=[c["name"] for c in synth.MBCONV_CONFIGS])
def test_mbconv_pattern(cfg, flags, record_err):
    """The pattern kernel: Fig. 5(d) (d kept in shared memory where the planner chooses it) and
    Fig. 5(c) (NO_PREFETCH: d through L2)."""
    g, feed, gy, ref = _case(cfg)
    plan = g.partition(L.device_query(0), flags)
    if flags:
        assert "Fig. 5(c)" in plan.describe()
    assert "pattern mbconv: " in plan.describe() and "not used" not in plan.describe().split("pattern mbconv")[1][:20]
    s = session(g, plan, feed, [gy])
    s.run()
    out = s.result(gy)
    s.run()                                   # a second launch reuses the workspace (barrier counters reset)
    record_err(rel_err(out, ref), 1e-4, module=cfg["name"], variant=f"pattern_{flags}")
    record_err(rel_err(s.result(gy), ref), 1e-4, module=cfg["name"], variant=f"pattern_{flags}_again")


@pytest.mark.parametrize("cfg", synth.MBCONV_CONFIGS, ids=[c["name"] for c in synth.MBCONV_CONFIGS])
def test_mbconv_generic(cfg, record_err):
    g, feed, gy, ref = _case(cfg)
    plan = g.partition(L.device_query(0), L.FLAG_NO_PATTERN)
    s = session(g, plan, feed, [gy])
    s.run()
    record_err(rel_err(s.result(gy), ref), 1e-4, module=cfg["name"], variant="generic_reuse")


@pytest.mark.parametrize("variant", ["a_unfused", "b_fused", "c_generic_global_sync"])
@pytest.mark.parametrize("idx", [0, 1, 3, 9])
def test_mbconv_fig5_variants(idx, variant, record_err):
    cfg = synth.MBCONV_CONFIGS[idx]
    g, feed, gy, ref = _case(cfg)
    plan = g.partition(L.device_query(0), VARIANTS[variant])
    s = session(g, plan, feed, [gy])
    s.run()
    record_err(rel_err(s.result(gy), ref), 1e-4, module=cfg["name"], variant=variant)
