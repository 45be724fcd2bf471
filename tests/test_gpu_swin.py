"""GPU parity for Swin-Transformer (Table 2) on the generic
fused-subprogram executor (the roll / window-partition index maps are folded into the GEMM loads
and stores, §6.2).  Tolerances as in test_gpu_parity.py: fp32 path rel 1e-4; bf16-operand path
max abs 2e-2 against the oracle's bf16-operand emulation."""
import numpy as np
import pytest

import synth.swin as S
from oracle import graphs as og
from oracle import te
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L
from paper_conf_asplos_xiazswwyfc24_b200 import models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session

pytestmark = pytest.mark.gpu


def rel_err(g, o):
    rms = np.sqrt(np.mean(o * o)) + 1e-30
    return float(np.max(np.abs(g - o) / np.maximum(np.abs(o), rms)))


def _run(cfg, flags=0, bf16=False):
    P = S.swin_params(cfg)
    fv = S.swin_feed_values(cfg, P)
    img = S.swin_input(cfg)
    g, names, x, y = M.swin(cfg)
    feed = {names[k]: v for k, v in fv.items()}
    feed[x] = img
    plan = g.partition(L.device_query(0), flags)
    s = session(g, plan, feed, [y])
    s.run()
    got = s.result(y)
    s.run()                                   # a second launch reuses the workspace
    again = s.result(y)
    spec, onames, ox, oy = og.swin(cfg)
    ref = te.evaluate(spec, feed, bf16_operands=bf16)[oy]
    return got, again, ref, plan


@pytest.mark.parametrize("batch", [1, 2])
@pytest.mark.parametrize("flags,cache", [(0, None), (L.FLAG_UNFUSED, None), (L.FLAG_NO_PREFETCH, None), (0, "2048")])
def test_swin_tiny_fp32(batch, flags, cache, monkeypatch):
    """Generic executor.  cache: SOUFFLE_CACHE_FLOATS -- 2048 floats hold one LayerNorm row block of
    x at a time, so the LRU scan spills tensors whose readers are still to come (§6.5)."""
    if cache:
        monkeypatch.setenv("SOUFFLE_CACHE_FLOATS", cache)
    got, again, ref, plan = _run(dict(S.SWIN_TINY, batch=batch), flags)
    if cache:
        assert "0 LRU eviction" not in plan.describe()
    assert rel_err(got, ref) <= 1e-4, plan.describe()[:2000]
    assert rel_err(again, ref) <= 1e-4


def test_swin_tiny_bf16_tensor_cores():
    """embed 64 so every Linear has K % 64 == 0 and runs on the tcgen05 GEMM stage."""
    cfg = dict(S.SWIN_TINY, embed=64, heads=(2, 4), gemm_dtype="bf16")
    got, again, ref, plan = _run(cfg, bf16=True)
    assert "GEMM_TC" in plan.describe()
    assert np.max(np.abs(got - ref)) <= 2e-2
    assert np.max(np.abs(again - ref)) <= 2e-2


# the Swin pattern kernels (kernels/swin.cu): head dim 32, window 7, C % 128 == 0.  56 x 56 images
# give a 14 x 14 stage (2 x 2 windows, shifted blocks with the mask), a patch merge and a 7 x 7
# stage whose window covers the map (no shift) -- every kernel and index map of the pattern
SWIN_PAT = dict(S.SWIN_TINY, embed=128, heads=(4, 8), gemm_dtype="bf16")


@pytest.mark.parametrize("batch", [1, 3])
def test_swin_pattern_small(batch, record_err):
    got, again, ref, plan = _run(dict(SWIN_PAT, batch=batch), bf16=True)
    assert "pattern swin: batch" in plan.describe()
    record_err(float(np.max(np.abs(got - ref))), 2e-2, batch=batch, rms=float(np.sqrt(np.mean(ref ** 2))))
    # split-K residual epilogues accumulate with fp32 atomics (order varies run to run): an ulp-level
    # difference can flip a later bf16 operand rounding, so repeat runs agree to a few bf16 ulps
    assert np.max(np.abs(got - again)) <= 5e-3


def test_swin_pattern_generic_agree():
    """The pattern kernels and the generic fused executor compute the same TE program."""
    cfg = dict(SWIN_PAT, batch=2)
    got, _, ref, plan = _run(cfg, bf16=True)
    gen, _, _, gplan = _run(cfg, flags=L.FLAG_NO_PATTERN, bf16=True)
    assert "pattern swin: batch" in plan.describe() and "pattern swin: not used" in gplan.describe()
    assert np.max(np.abs(got - gen)) <= 2e-2


def _swin_b_child(batch):
    got, again, ref, plan = _run(dict(S.SWIN_B, batch=batch), bf16=True)
    print("RESULT", got.shape[0], got.shape[1], float(np.max(np.abs(got - ref))), float(np.max(np.abs(again - ref))),
          float(np.sqrt(np.mean(ref ** 2))), "pattern swin: batch" in plan.describe())


@pytest.mark.parametrize("batch,two_sm", [(1, False), (8, False), (8, True)])
def test_swin_b_full_size(batch, two_sm, record_err):
    """Full Swin-B (BASELINE.json configs[4]) at batch 1 and 8 through the pattern kernels against the
    bf16-operand oracle, in a fresh process (isolated from the kernels the other tests ran); batch 8
    also with the opt-in 2-SM (cta_group::2) GEMM tiles, which its stage-1/2 GEMMs select."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = "import sys; sys.path.insert(0, %r); sys.path.insert(0, %r); import test_gpu_swin as t; t._swin_b_child(%d)" % (
        root, os.path.join(root, "tests"), batch)
    env = dict(os.environ)
    if two_sm:
        env["SOUFFLE_SWIN_2SM"] = "1"
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=900, cwd=root, env=env)
    line = [ln for ln in r.stdout.splitlines() if ln.startswith("RESULT")]
    assert line, r.stderr[-2000:]
    _, b, n, e1, e2, rms, pat = line[0].split()
    assert (int(b), int(n)) == (batch, 1000) and pat == "True"
    assert float(e2) <= 2e-2
    record_err(float(e1), 2e-2, batch=batch, rms=float(rms), two_sm=two_sm)


def _swin_b64_child():
    """Swin-B at batch 64 (the per-GPU batch of the bench's 64-image replica job, 2-SM GEMM tiles)
    against the oracle on sampled images: every image is independent, so the oracle evaluates the
    batch-1 program on images 0, 37 and 63 only."""
    cfg = dict(S.SWIN_B, batch=64)
    P = S.swin_params(cfg)
    fv = S.swin_feed_values(cfg, P)
    img = S.swin_input(cfg)
    g, names, x, y = M.swin(cfg)
    feed = {names[k]: v for k, v in fv.items()}
    feed[x] = img
    plan = g.partition(L.device_query(0))
    s = session(g, plan, feed, [y])
    s.run()
    got = s.result(y)
    c1 = dict(S.SWIN_B, batch=1)
    spec, onames, ox, oy = og.swin(c1)
    errs = []
    for i in (0, 37, 63):
        f1 = {onames[k]: v for k, v in S.swin_feed_values(c1, S.swin_params(c1)).items()}
        f1[ox] = img[i:i + 1]
        ref = te.evaluate(spec, f1, bf16_operands=True)[oy]
        errs.append(float(np.max(np.abs(got[i] - ref[0]))))
    print("RESULT", max(errs), "pattern swin: batch 64" in plan.describe())


def test_swin_b_batch64_sampled(record_err):
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = "import sys; sys.path.insert(0, %r); sys.path.insert(0, %r); import test_gpu_swin as t; t._swin_b64_child()" % (
        root, os.path.join(root, "tests"))
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=900, cwd=root)
    line = [ln for ln in r.stdout.splitlines() if ln.startswith("RESULT")]
    assert line, r.stderr[-2000:]
    _, err, pat = line[0].split()
    assert pat == "True"
    record_err(float(err), 2e-2, batch=64, sampled_images=[0, 37, 63])
