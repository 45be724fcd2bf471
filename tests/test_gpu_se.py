"""GPU parity of the EfficientNet squeeze-and-excitation sub-modules M0-M9 (Fig. 5 / 6,
L1511-1564) against the fp64 oracle: the pattern kernel with and without the shared-memory data
reuse (Fig. 5(d) / (c)), the generic fused executor and the unfused V0 path.  fp32 everywhere:
max_i |g - o| / max(|o|, rms(o)) <= 1e-4."""
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
    rms = np.sqrt(np.mean(o * o)) + 1e-30
    return float(np.max(np.abs(g - o) / np.maximum(np.abs(o), rms)))


@pytest.mark.parametrize("flags", [0, L.FLAG_NO_PREFETCH, L.FLAG_NO_PATTERN, L.FLAG_UNFUSED],
                         ids=["pattern_reuse", "pattern_no_reuse", "generic", "unfused"])
@pytest.mark.parametrize("cfg", synth.SE_CONFIGS, ids=[c["name"] for c in synth.SE_CONFIGS])
def test_se_module(cfg, flags, record_err):
    x = synth.se_input(cfg)
    p = synth.se_params(cfg)
    spec, names, X, Y = og.se_module(cfg)
    feed = {names[k]: v for k, v in p.items()}
    feed[X] = x
    ref = te.evaluate(spec, feed)[Y]
    g, gnames, gx, gy = M.se_module(cfg)
    plan = g.partition(L.device_query(0), flags)
    if flags in (0, L.FLAG_NO_PREFETCH):
        assert "pattern se: squeeze-excitation" in plan.describe()
    s = session(g, plan, {gnames[k]: p[k] for k in p} | {gx: x}, [gy])
    s.run()
    out = s.result(gy)
    s.run()                                   # a second launch reuses the workspace
    again = s.result(gy)
    record_err(rel_err(out, ref), 1e-4, module=cfg["name"], flags=int(flags))
    if flags in (0, L.FLAG_NO_PREFETCH):
        assert np.array_equal(out, again)     # fixed-order reductions: bit-reproducible
    else:
        assert rel_err(again, ref) <= 1e-4
