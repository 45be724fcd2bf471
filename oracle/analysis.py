"""Oracle: Souffle's global analysis and partitioning, restated from the paper in plain Python.

TEST INFRASTRUCTURE ONLY (see oracle/te.py header).  The C++ library must agree with every
function here BIT-EXACTLY (integers only).  Each function cites the passage it follows; the
readings taken where the paper is silent or garbled are listed in DESIGN.md §"Readings".

  classify()        §5.2 L860-895 (one-relies-on-one vs one-relies-on-many) and §5.3
                    (compute/memory ratio, threshold 3).
  reuse_sets()      §5.1: s(t_i) = {op_j..op_k}; spatial vs temporal L820-858.
  bfs_order()       Alg. 1 line 2 "BFS(P)" L1258 -- reading: Kahn's algorithm, FIFO queue.
  partition()       §5.4, Alg. 1 lines 2-9 L1257-1269, Fig. 2 L682-699.
  index_map()       §5.2 Eq. 1 L897-919 and §6.2 Eq. 2 L1086-1153 -- composition by substitution
                    (consumer map applied first), enumerated as flat source offsets.
  levels(), hgroups()  §6.1 L1062-1084 horizontal transformation candidates (reading in DESIGN.md).
"""
from __future__ import annotations

import math
from collections import deque

from .te import infer_shapes

OR_OPS = {"ew", "reshape", "permute", "slice", "roll"}
MR_OPS = {"matmul", "reduce"}


def numel(s):
    return math.prod(s)


def te_inputs(n):
    op = n["op"]
    if op == "placeholder":
        return []
    if op == "matmul":
        return [n["a"], n["b"]]
    if op == "ew":
        return list(n["in"])
    return [n["in"]]


def classify(spec):
    """Per node: dict(dep=0 OR /1 MR /-1 placeholder, ops, accesses, ci=0/1).

    ops (§5.3 "number of arithmetic instructions"): matmul 2*K per output element (mul and add
    counted separately); reduce R per output element (R = reduce extent); elementwise 1 per
    output element; reshape/permute/slice 0.
    accesses ("per tensor element that is both read and written"): |out| + sum over DISTINCT input
    tensors of the distinct elements read (= numel(input), except a strided slice reads |out|).
    CI iff ops >= 3 * accesses (ratio < 3 -> memory-intensive, L949-951)."""
    shapes = infer_shapes(spec)
    info = []
    for i, n in enumerate(spec["nodes"]):
        op = n["op"]
        if op == "placeholder":
            info.append(dict(dep=-1, ops=0, accesses=0, ci=0))
            continue
        O = numel(shapes[i])
        if op == "matmul":
            K = shapes[n["a"]][-1]
            ops = 2 * K * O
        elif op == "reduce":
            ops = shapes[n["in"]][n["axis"] % len(shapes[n["in"]])] * O
        elif op == "ew":
            ops = O
        else:
            ops = 0
        acc = O
        for j in sorted(set(te_inputs(n))):
            acc += O if op == "slice" else numel(shapes[j])
        info.append(dict(dep=1 if op in MR_OPS else 0, ops=ops, accesses=acc, ci=1 if ops >= 3 * acc else 0))
    return info


def consumers(spec):
    cons = [[] for _ in spec["nodes"]]
    for i, n in enumerate(spec["nodes"]):
        for j in sorted(set(te_inputs(n))):
            cons[j].append(i)
    return cons


def reachability(spec):
    """reach[i] = bitmask (Python int) of the nodes reachable from i (its descendants)."""
    cons = consumers(spec)
    reach = [0] * len(spec["nodes"])
    for i in reversed(range(len(spec["nodes"]))):
        m = 0
        for c in cons[i]:
            m |= (1 << c) | reach[c]
        reach[i] = m
    return reach


def reuse_sets(spec):
    """{t: (sorted consumer TE ids, kind)} for every tensor read by >= 2 TEs (§5.1).
    kind 0 = spatial (consumers pairwise independent -> horizontal, §6.1), 1 = temporal."""
    cons = consumers(spec)
    reach = reachability(spec)
    out = {}
    for t, cs in enumerate(cons):
        if len(cs) < 2:
            continue
        dep = any((reach[a] >> b) & 1 or (reach[b] >> a) & 1 for x, a in enumerate(cs) for b in cs[x + 1:])
        out[t] = (sorted(cs), 1 if dep else 0)
    return out


def bfs_order(spec):
    """Kahn's algorithm with a FIFO queue over TE->TE edges (placeholders are not TEs).
    Seeds: TEs with no TE predecessor in ascending id; successors released in ascending id."""
    nodes = spec["nodes"]
    is_te = [n["op"] != "placeholder" for n in nodes]
    preds = [sorted({j for j in te_inputs(n) if is_te[j]}) for n in nodes]
    succ = [[] for _ in nodes]
    for i, ps in enumerate(preds):
        for j in ps:
            succ[j].append(i)
    indeg = [len(p) for p in preds]
    q = deque(i for i in range(len(nodes)) if is_te[i] and indeg[i] == 0)
    order = []
    while q:
        e = q.popleft()
        order.append(e)
        for s in sorted(succ[e]):
            indeg[s] -= 1
            if indeg[s] == 0:
                q.append(s)
    return order


def occupancy(dev, smem, regs, threads):
    lim = [dev["max_blocks_per_sm"]]
    if smem > 0:
        lim.append(dev["smem_per_sm"] // (smem + dev["smem_reserved_per_block"]))
    if regs * threads > 0:
        lim.append(dev["regs_per_sm"] // (regs * threads))
    if threads > 0:
        lim.append(dev["max_threads_per_sm"] // threads)
    return min(lim)


def fits(dev, r):
    """r = (grid, smem, regs, threads) maxima over the CI TEs of the candidate subprogram.
    rule 1 (paper, §5.4): max_grid * max_occ <= C, occupancy = shared memory bytes
        (Fig. 2: 48 KB capacity, 1 KB per block; '<=' per Fig. 2 'at most 48 blocks', L668).
    rule 0 (B200-exact): max_grid <= num_sms * blocks-per-SM(smem, regs*threads, threads)."""
    grid, smem, regs, threads = r
    if dev["rule"] == 1:
        return grid * smem <= dev["capacity_C"]
    return grid <= dev["num_sms"] * occupancy(dev, smem, regs, threads)


def partition(spec, resources, dev, order=None, info=None):
    """Greedy resource-aware partition (Alg. 1 lines 2-9; §5.4).  Only CI TEs can open a new
    subprogram (L984-993); MI TEs always join the current one.  A CI TE e forms the candidate
    maxima; if the current SP already holds a CI TE and the candidate does not fit, a new SP
    starting with e is opened (L1009-1011).  resources[e] = (grid, smem, regs, threads).
    Returns te_to_sp list (-1 for placeholders)."""
    info = info or classify(spec)
    order = order if order is not None else bfs_order(spec)
    assign = [-1] * len(spec["nodes"])
    sp = 0
    cur = None
    for e in order:
        if info[e]["ci"]:
            r = tuple(resources[e])
            if cur is None:
                cur = r
            else:
                cand = tuple(max(a, b) for a, b in zip(cur, r))
                if fits(dev, cand):
                    cur = cand
                else:
                    sp += 1
                    cur = r
        assign[e] = sp
    return assign


# ---------------------------------------------------------------- index maps (§5.2 / §6.2)
def _unravel(flat, shape):
    idx = []
    for d in reversed(shape):
        idx.append(flat % d)
        flat //= d
    return list(reversed(idx))


def _ravel(idx, shape):
    f = 0
    for d, v in zip(shape, idx):
        f = f * d + v
    return f


def or_map(n, shapes, i, j_pos, idx):
    """Map an output index of OR TE i to the index in its j_pos-th input (Eq. 1, quasi-affine)."""
    op = n["op"]
    if op == "ew":
        ish = shapes[n["in"][j_pos]]
        off = len(idx) - len(ish)
        return [0 if ish[d] == 1 else idx[d + off] for d in range(len(ish))]
    if op == "reshape":
        return _unravel(_ravel(idx, shapes[i]), shapes[n["in"]])
    if op == "permute":
        src = [0] * len(idx)
        for k, p in enumerate(n["perm"]):
            src[p] = idx[k]
        return src
    if op == "slice":
        return [b + v * s for b, v, s in zip(n["begin"], idx, n["stride"])]
    if op == "roll":   # quasi-affine: (i - shift) mod n
        return [(v - sh) % d for v, sh, d in zip(idx, n["shifts"], shapes[i])]
    raise ValueError(op)


def or_path(spec, t, s):
    """Input positions of the first OR-only path from TE t back to tensor s (operand order,
    depth-first), or None."""
    if t == s:
        return []
    n = spec["nodes"][t]
    if n["op"] not in OR_OPS:
        return None
    ins = n["in"] if n["op"] == "ew" else [n["in"]]
    for pos, j in enumerate(ins):
        sub = or_path(spec, j, s)
        if sub is not None:
            return [(t, pos)] + sub
    return None


def index_map(spec, t, s):
    """Flat source offset in s for every element of t (row-major), composing the per-TE maps by
    substitution: src = f_0(f_1(...f_{n-1}(v))) -- the consumer's map is applied first.
    (Eq. 2 prints the reverse order and Fig. 4 prints A[j,2i]; substitution gives A[2j,i].)
    Returns None if no OR-only path exists."""
    shapes = infer_shapes(spec)
    path = or_path(spec, t, s)
    if path is None:
        return None
    out = []
    for f in range(numel(shapes[t])):
        idx = _unravel(f, shapes[t])
        for node, pos in path:
            idx = or_map(spec["nodes"][node], shapes, node, pos, idx)
        out.append(_ravel(idx, shapes[s]))
    return out


# ---------------------------------------------------------------- horizontal candidates (§6.1)
def levels(spec):
    """ASAP level: 0 for TEs without TE predecessors, else 1 + max(level of TE predecessors)."""
    lv = [-1] * len(spec["nodes"])
    for i, n in enumerate(spec["nodes"]):
        if n["op"] == "placeholder":
            continue
        ps = [lv[j] for j in te_inputs(n) if spec["nodes"][j]["op"] != "placeholder"]
        lv[i] = 0 if not ps else 1 + max(ps)
    return lv


def hgroups(spec, assign):
    """Horizontal groups of matmul TEs (§6.1): same subprogram, same level (so the group DAG stays
    acyclic and the members are independent), same reduce extent K and precision.
      pass 1 (spatial reuse, L1071-1076): members that share the A operand and trans_b -> concat
              along N; a group needs >= 2 members.
      pass 2 (Fig. 3): remaining 2-D matmuls with equal (K, N) -> concat along M.
    Returns group id per node (-1 if not grouped), ids dense in first-member order, and the kind
    per group (0 = N-concat, 1 = M-concat)."""
    shapes = infer_shapes(spec)
    lv = levels(spec)
    nodes = spec["nodes"]
    mm = [i for i, n in enumerate(nodes) if n["op"] == "matmul"]
    gid = [-1] * len(nodes)
    groups = []

    def K(i):
        return shapes[nodes[i]["a"]][-1]

    for i in mm:
        if gid[i] >= 0:
            continue
        n = nodes[i]
        mem = [j for j in mm if j > i and gid[j] < 0 and assign[j] == assign[i] and lv[j] == lv[i]
               and nodes[j]["a"] == n["a"] and nodes[j]["trans_b"] == n["trans_b"]
               and nodes[j]["prec"] == n["prec"] and K(j) == K(i)
               and len(shapes[nodes[j]["b"]]) == len(shapes[n["b"]])]
        if mem:
            g = len(groups)
            groups.append(0)
            for j in [i] + mem:
                gid[j] = g
    for i in mm:
        if gid[i] >= 0 or len(shapes[i]) != 2:
            continue
        n = nodes[i]
        mem = [j for j in mm if j > i and gid[j] < 0 and len(shapes[j]) == 2 and assign[j] == assign[i]
               and lv[j] == lv[i] and nodes[j]["prec"] == n["prec"] and K(j) == K(i)
               and shapes[j][1] == shapes[i][1]]
        if mem:
            g = len(groups)
            groups.append(1)
            for j in [i] + mem:
                gid[j] = g
    return gid, groups
