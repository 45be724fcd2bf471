"""Pins for the oracle's analysis (CPU only): the paper's worked examples (Fig. 2/3/4, Eq. 1,
Table 5 kernel counts) and brute-force properties."""
import json
import os

import numpy as np
import pytest

import synth
from oracle import analysis as an
from oracle import graphs, te, transforms

GOLD = os.path.join(os.path.dirname(__file__), "golden")

PAPER_DEV = dict(rule=1, capacity_C=48 * 1024, num_sms=0, smem_per_sm=0, smem_reserved_per_block=0,
                 regs_per_sm=0, max_threads_per_sm=0, max_blocks_per_sm=0)
B200 = dict(rule=0, capacity_C=0, num_sms=148, smem_per_sm=233472, smem_reserved_per_block=1024,
            regs_per_sm=65536, max_threads_per_sm=2048, max_blocks_per_sm=32)


def test_fig2_classification_reuse_partition():
    g = json.load(open(os.path.join(GOLD, "fig2.json")))
    spec, ids = graphs.fig2()
    info = an.classify(spec)
    for name, (dep, inten) in g["classification"].items():
        i = ids[name]
        assert info[i]["dep"] == (1 if dep == "MR" else 0), name
        assert info[i]["ci"] == (1 if inten == "CI" else 0), name
    # ratios from the reading in DESIGN.md: 42.7 and 56.9
    assert abs(info[ids["TE0"]]["ops"] / info[ids["TE0"]]["accesses"] - 42.67) < 0.01
    assert abs(info[ids["TE4"]]["ops"] / info[ids["TE4"]]["accesses"] - 56.89) < 0.01
    reuse = an.reuse_sets(spec)
    assert reuse[ids["TE0"]] == ([ids["TE1"], ids["TE3"]], 1)       # temporal: TE1 -> TE2 -> TE3
    res = {i: (0, 0, 0, 0) for i in range(len(spec["nodes"]))}
    for name, r in g["paper_resources"].items():
        res[ids[name]] = (r["grid"], r["smem"], 0, 0)
    assign = an.partition(spec, res, PAPER_DEV)
    got = {}
    for name in ("TE0", "TE1", "TE2", "TE3", "TE4"):
        got.setdefault(assign[ids[name]], []).append(name)
    assert [got[k] for k in sorted(got)] == g["partition"]


def test_partition_inequality_is_inclusive_at_capacity():
    """Reading (ii): '<=' -- a subprogram whose max_grid*max_smem equals C exactly still fits."""
    spec, ids = graphs.fig2()
    res = {i: (0, 0, 0, 0) for i in range(len(spec["nodes"]))}
    res[ids["TE0"]] = (16, 1024, 0, 0)
    res[ids["TE2"]] = (16, 1024, 0, 0)
    res[ids["TE4"]] = (48, 1024, 0, 0)
    assert len(set(a for a in an.partition(spec, res, PAPER_DEV) if a >= 0)) == 1
    res[ids["TE4"]] = (49, 1024, 0, 0)
    assert len(set(a for a in an.partition(spec, res, PAPER_DEV) if a >= 0)) == 2


def test_eq1_identity_map_and_mr_region():
    spec, ids = graphs.fig2()
    m = an.index_map(spec, ids["TE1"], ids["TE0"])    # R1: O1[i,j] -> O0[i,j], M = I2, c = 0
    assert m == list(range(64 * 64))
    assert an.index_map(spec, ids["TE2"], ids["TE1"]) is None    # MR: no one-to-one map


def test_fig4_vertical_map_corrected():
    g = json.load(open(os.path.join(GOLD, "fig4.json")))
    spec, ids = graphs.fig4()
    assert an.index_map(spec, ids["D"], ids["A"]) == g["D_to_A_flat_offsets_row_major"]
    A = synth.normal(2, (4, 8))
    vals = te.evaluate(spec, {ids["A"]: A})
    fused = transforms.vfused_eval(spec, vals, ids["D"], leaves={ids["A"]})
    assert np.array_equal(fused, vals[ids["D"]])


def test_fig3_horizontal_mconcat_equals_unfused():
    spec, ids = graphs.fig3()
    ins = synth.spec_inputs(spec, 4, integer=True)
    vals = te.evaluate(spec, ins)
    fused = transforms.hfused_mconcat([ins[ids["A1"]], ins[ids["A2"]]], [ins[ids["B1"]], ins[ids["B2"]]])
    assert fused.shape == (6, 16)
    assert np.array_equal(fused[:4], vals[ids["C1"]]) and np.array_equal(fused[4:], vals[ids["C2"]])
    assign = an.partition(spec, {i: (1, 0, 0, 0) for i in range(len(spec["nodes"]))}, B200)
    gid, kinds = an.hgroups(spec, assign)
    assert gid[ids["C1"]] == gid[ids["C2"]] == 0 and kinds == [1]


def test_bert_qkv_nconcat_and_reuse():
    cfg = synth.BERT_TINY
    spec, X, plist, y = graphs.bert(cfg, layers=1)
    reuse = an.reuse_sets(spec)
    cons, kind = reuse[X]
    mm = [i for i in cons if spec["nodes"][i]["op"] == "matmul"]
    assert len(mm) == 3 and kind == 1           # X also feeds the residual add -> temporal overall
    assign = [0 if n["op"] != "placeholder" else -1 for n in spec["nodes"]]
    gid, kinds = an.hgroups(spec, assign)
    assert len({gid[i] for i in mm}) == 1 and kinds[gid[mm[0]]] == 0
    ins = synth.spec_inputs(spec, 1, integer=True)
    vals = te.evaluate(spec, ins)
    Ws = [ins[spec["nodes"][i]["b"]] for i in mm]
    fused = transforms.hfused_nconcat(ins[X], Ws)
    H = cfg["hidden"]
    for k, i in enumerate(mm):
        assert np.array_equal(fused[:, k * H:(k + 1) * H], vals[i])


def test_bert_head_scatter_map_and_classification():
    cfg = synth.BERT_BASE
    spec, X, plist, y = graphs.bert(cfg, layers=1)
    info = an.classify(spec)
    mm = [i for i, n in enumerate(spec["nodes"]) if n["op"] == "matmul"]
    assert all(info[i]["ci"] for i in mm)                  # S=128 GEMMs are compute-intensive
    assert abs(info[mm[0]]["ops"] / info[mm[0]]["accesses"] - 192.0) < 1e-9   # 2*768*98304 / (98304+98304+589824)
    Qp = next(i for i, n in enumerate(spec["nodes"]) if n["op"] == "permute")
    Q1 = spec["nodes"][spec["nodes"][Qp]["in"]]["in"]
    m = an.index_map(spec, Qp, Q1)                          # [nh,S,d] -> [S,H]
    S, H, d = 128, 768, 64
    for f in (0, 1, 63, 64, 8191, 8192, 12 * S * d - 1):
        h, s, dd = f // (S * d), (f // d) % S, f % d
        assert m[f] == s * H + h * d + dd


def test_table5_lstm_and_mmoe_are_one_subprogram():
    """Table 5 (L1466, L1469): LSTM and MMoE compile to ONE kernel.  With the ratio-3 rule every
    batch-1 GEMV is memory-intensive, so no CI TE can split."""
    cfg = dict(synth.LSTM_CFG, steps=5)
    spec, *_ = graphs.lstm(cfg)
    info = an.classify(spec)
    assert not any(x["ci"] for x in info)
    assign = an.partition(spec, {i: (1, 0, 0, 0) for i in range(len(spec["nodes"]))}, B200)
    assert {a for a in assign if a >= 0} == {0}
    spec, *_ = graphs.mmoe(synth.MMOE_CFG)
    info = an.classify(spec)
    assert not any(x["ci"] for x in info)
    assign = an.partition(spec, {}, B200)
    assert {a for a in assign if a >= 0} == {0}


def _brute_topological(spec, order):
    pos = {e: k for k, e in enumerate(order)}
    for i, n in enumerate(spec["nodes"]):
        for j in an.te_inputs(n):
            if spec["nodes"][j]["op"] != "placeholder":
                assert pos[j] < pos[i]


@pytest.mark.parametrize("seed", range(20))
def test_order_is_topological_and_partition_properties(seed):
    spec = synth.random_spec(seed, n_ops=25)
    order = an.bfs_order(spec)
    n_te = sum(1 for n in spec["nodes"] if n["op"] != "placeholder")
    assert sorted(order) == [i for i, n in enumerate(spec["nodes"]) if n["op"] != "placeholder"]
    assert len(order) == n_te
    _brute_topological(spec, order)
    r = synth.rng(seed)
    res = {i: (int(r.integers(1, 300)), int(r.integers(0, 3)) * 32768, 64, 256) for i in range(len(spec["nodes"]))}
    assign = an.partition(spec, res, B200)
    info = an.classify(spec)
    # subprogram ids are non-decreasing along the order, start at 0, and each new SP starts at a CI TE
    last = 0
    for k, e in enumerate(order):
        assert assign[e] in (last, last + 1)
        if assign[e] == last + 1:
            assert info[e]["ci"]
        last = assign[e]
    # brute check: each SP's CI resource maxima fit, unless the SP holds a single CI TE
    for sp in set(a for a in assign if a >= 0):
        cis = [e for e in order if assign[e] == sp and info[e]["ci"]]
        if len(cis) > 1:
            mx = tuple(max(res[e][k] for e in cis) for k in range(4))
            assert an.fits(B200, mx)


# ---------------------------------------------------------------- BFS order and reuse kind pins
def _golden_bfs_spec():
    g = json.load(open(os.path.join(GOLD, "bfs_order.json")))
    b = graphs.SpecBuilder()
    for nd in g["dag"]["nodes"]:
        if nd.get("op") == "placeholder":
            b.ph((4, 8), const=0)
        else:
            b.ew(nd["fn"], *nd["in"])
    for o in g["dag"]["outputs"]:
        b.out(o)
    return b.spec(), g


def _kahn(spec, lifo=False, release_desc=False):
    """Deliberately WRONG variants of the order, to show the golden distinguishes them."""
    nodes = spec["nodes"]
    is_te = [n["op"] != "placeholder" for n in nodes]
    preds = [sorted({j for j in an.te_inputs(n) if is_te[j]}) for n in nodes]
    succ = [[] for _ in nodes]
    for i, ps in enumerate(preds):
        for j in ps:
            succ[j].append(i)
    indeg = [len(p) for p in preds]
    q = [i for i in range(len(nodes)) if is_te[i] and indeg[i] == 0]
    order = []
    while q:
        e = q.pop() if lifo else q.pop(0)
        order.append(e)
        for s in sorted(succ[e], reverse=release_desc):
            indeg[s] -= 1
            if indeg[s] == 0:
                q.append(s)
    return order


def test_bfs_order_hand_derived_golden():
    """Alg. 1 line 2 'BFS(P)' (L1258), reading R3: Kahn + FIFO.  The golden order was derived by hand
    (tests/golden/bfs_order.json 'derivation'); a LIFO queue or descending successor release fails."""
    spec, g = _golden_bfs_spec()
    assert an.bfs_order(spec) == g["order"]
    _brute_topological(spec, g["order"])
    assert _kahn(spec, lifo=True) == g["wrong_orders"]["lifo_stack_kahn"] != g["order"]
    assert _kahn(spec, release_desc=True) == g["wrong_orders"]["successors_released_descending"] != g["order"]
    # breadth-first property: every TE appears after all TEs of a strictly smaller ASAP level that
    # were enqueued before it -- here simply: levels are non-decreasing along the FIFO order
    lv = an.levels(spec)
    assert [lv[e] for e in g["order"]] == sorted(lv[e] for e in g["order"])


def _qkv_spec(chain):
    b = graphs.SpecBuilder()
    X = b.ph((16, 32), const=0)
    Wq = b.ph((32, 32))
    Q = b.mm(X, Wq)
    Wk = b.ph((32, 32))
    K = b.mm(X, Wk)
    src = X
    XK = None
    if chain:
        XK = b.ew("add", X, K)
        src = XK
    Wv = b.ph((32, 32))
    V = b.mm(src, Wv)
    for t in (Q, K, V):
        b.out(t)
    return b.spec(), dict(X=X, Q=Q, K=K, V=V, XK=XK)


def test_reuse_kind_spatial_for_independent_qkv():
    """Fig. 1(a) / §5.1: Q, K, V GEMMs sharing X with no path between them -> spatial (0);
    making one consumer depend on another turns the set temporal (1)."""
    g = json.load(open(os.path.join(GOLD, "reuse_spatial.json")))["programs"]
    spec, ids = _qkv_spec(chain=False)
    e = g["qkv"]["expected"]
    assert an.reuse_sets(spec)[ids[e["tensor"]]] == ([ids[c] for c in e["consumers"]], e["kind"]) == ([2, 4, 6], 0)
    spec, ids = _qkv_spec(chain=True)
    e = g["qkv_chain"]["expected"]
    assert an.reuse_sets(spec)[ids[e["tensor"]]] == (sorted(ids[c] for c in e["consumers"]), e["kind"])
    # the spatial set is also the horizontal group (§6.1): one N-concat group of 3
    spec, ids = _qkv_spec(chain=False)
    gid, kinds = an.hgroups(spec, [0 if n["op"] != "placeholder" else -1 for n in spec["nodes"]])
    assert gid[ids["Q"]] == gid[ids["K"]] == gid[ids["V"]] == 0 and kinds == [0]
