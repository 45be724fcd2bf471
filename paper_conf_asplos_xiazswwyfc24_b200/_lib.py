"""Thin ctypes binding of libsouffle (include/souffle.h).  Argument marshalling only: every step of
the path runs in the C++ library and its sm_100a kernels.  Functions keep the C names."""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libsouffle.so")

F32, BF16 = 0, 1
OP_PLACEHOLDER, OP_MATMUL, OP_ELEMENTWISE, OP_REDUCE, OP_RESHAPE, OP_PERMUTE, OP_SLICE, OP_ROLL = range(8)
EW = dict(add=0, sub=1, mul=2, div=3, max=4, exp=5, tanh=6, sigmoid=7, relu=8, gelu_erf=9, rsqrt=10, neg=11,
          add_scalar=12, mul_scalar=13)
RED = dict(sum=0, max=1, mean=2)
FLAG_UNFUSED, FLAG_NO_HORIZONTAL, FLAG_NO_VERTICAL, FLAG_NO_GLOBAL_SYNC, FLAG_NO_PREFETCH, FLAG_NO_LN_REWRITE = (
    1, 2, 4, 8, 16, 32)
FLAG_NO_PATTERN = 64

ERRORS = {1: "INVALID_ARG", 2: "SHAPE", 3: "UNSUPPORTED", 4: "RESOURCE", 5: "CUDA", 6: "STATE", 7: "OOM"}


class SouffleError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"souffle error {code} ({ERRORS.get(code, '?')}): {msg}")
        self.code = code


class DeviceDesc(C.Structure):
    _fields_ = [("num_sms", C.c_int32), ("smem_per_sm", C.c_int64), ("smem_per_block_max", C.c_int64),
                ("smem_reserved_per_block", C.c_int64), ("regs_per_sm", C.c_int32),
                ("max_threads_per_sm", C.c_int32), ("max_blocks_per_sm", C.c_int32), ("rule", C.c_int32),
                ("capacity_C", C.c_int64)]


# name -> (restype is status, argtypes)
_SIGS = {
    "souffle_graph_create": [C.POINTER(C.c_void_p)],
    "souffle_graph_destroy": [C.c_void_p],
    "souffle_placeholder": [C.c_void_p, C.c_int32, C.POINTER(C.c_int64), C.c_int32, C.c_int32, C.POINTER(C.c_int32)],
    "souffle_matmul": [C.c_void_p, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.POINTER(C.c_int32)],
    "souffle_elementwise": [C.c_void_p, C.c_int32, C.c_int32, C.POINTER(C.c_int32), C.c_double, C.POINTER(C.c_int32)],
    "souffle_reduce": [C.c_void_p, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.POINTER(C.c_int32)],
    "souffle_reshape": [C.c_void_p, C.c_int32, C.c_int32, C.POINTER(C.c_int64), C.POINTER(C.c_int32)],
    "souffle_permute": [C.c_void_p, C.c_int32, C.POINTER(C.c_int32), C.POINTER(C.c_int32)],
    "souffle_roll": [C.c_void_p, C.c_int32, C.POINTER(C.c_int64), C.POINTER(C.c_int32)],
    "souffle_slice": [C.c_void_p, C.c_int32, C.POINTER(C.c_int64), C.POINTER(C.c_int64), C.POINTER(C.c_int64),
                      C.POINTER(C.c_int32)],
    "souffle_mark_output": [C.c_void_p, C.c_int32],
    "souffle_graph_num_nodes": [C.c_void_p, C.POINTER(C.c_int32)],
    "souffle_graph_node": [C.c_void_p, C.c_int32, C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_int64),
                           C.POINTER(C.c_int32)],
    "souffle_set_te_resources": [C.c_void_p, C.c_int32, C.c_int64, C.c_int64, C.c_int32, C.c_int32],
    "souffle_device_query": [C.c_int32, C.POINTER(DeviceDesc)],
    "souffle_device_b200": [C.POINTER(DeviceDesc)],
    "souffle_partition": [C.c_void_p, C.POINTER(DeviceDesc), C.c_uint32, C.POINTER(C.c_void_p)],
    "souffle_plan_destroy": [C.c_void_p],
    "souffle_plan_num_nodes": [C.c_void_p, C.POINTER(C.c_int32)],
    "souffle_plan_num_tes": [C.c_void_p, C.POINTER(C.c_int32)],
    "souffle_plan_num_subprograms": [C.c_void_p, C.POINTER(C.c_int32)],
    "souffle_plan_assignment": [C.c_void_p, C.POINTER(C.c_int32)],
    "souffle_plan_bfs_order": [C.c_void_p, C.POINTER(C.c_int32)],
    "souffle_plan_te_info": [C.c_void_p, C.c_int32, C.POINTER(C.c_int32), C.POINTER(C.c_int32),
                             C.POINTER(C.c_int64), C.POINTER(C.c_int64), C.POINTER(C.c_int64), C.POINTER(C.c_int64),
                             C.POINTER(C.c_int32), C.POINTER(C.c_int32)],
    "souffle_plan_reuse_set": [C.c_void_p, C.c_int32, C.POINTER(C.c_int32), C.c_int32, C.POINTER(C.c_int32),
                               C.POINTER(C.c_int32)],
    "souffle_plan_index_map": [C.c_void_p, C.c_int32, C.c_int32, C.POINTER(C.c_int64)],
    "souffle_plan_hgroup": [C.c_void_p, C.c_int32, C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_int32)],
    "souffle_plan_exec_info": [C.c_void_p, C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_int32)],
    "souffle_plan_describe": [C.c_void_p, C.POINTER(C.c_char_p)],
    "souffle_plan_workspace_bytes": [C.c_void_p, C.POINTER(C.c_size_t)],
    "souffle_bind": [C.c_void_p, C.c_int32, C.c_void_p],
    "souffle_workspace_init": [C.c_void_p, C.c_void_p, C.c_void_p],
    "souffle_run": [C.c_void_p, C.c_void_p, C.c_void_p],
    "souffle_plan_set_profiling": [C.c_void_p, C.c_int32],
    "souffle_plan_read_profile": [C.c_void_p, C.c_void_p, C.POINTER(C.c_double), C.c_int32, C.POINTER(C.c_int32)],
}
EXPORTS = sorted(list(_SIGS) + ["souffle_last_error", "souffle_version"])

_lib = None


def load(build_if_missing=True):
    """Load libsouffle.so (build it in-tree with nvcc first if it is missing)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        if not build_if_missing:
            raise OSError(f"{LIB_PATH} missing; run python -m paper_conf_asplos_xiazswwyfc24_b200.build")
        from .build import build
        build()
    lib = C.CDLL(LIB_PATH)
    for name, args in _SIGS.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = C.c_int32
    lib.souffle_last_error.restype = C.c_char_p
    lib.souffle_last_error.argtypes = []
    lib.souffle_version.restype = C.c_char_p
    lib.souffle_version.argtypes = []
    _lib = lib
    return lib


def check(status):
    if status != 0:
        raise SouffleError(status, load().souffle_last_error().decode())


def _i64(seq):
    seq = [int(x) for x in seq]
    return (C.c_int64 * max(1, len(seq)))(*seq)


def _i32(seq):
    seq = [int(x) for x in seq]
    return (C.c_int32 * max(1, len(seq)))(*seq)


class Graph:
    """TE-program builder over the C ABI (souffle_graph_create / TE ops / souffle_mark_output)."""

    def __init__(self):
        self.lib = load()
        h = C.c_void_p()
        check(self.lib.souffle_graph_create(C.byref(h)))
        self.h = h
        self.outputs = []

    def __del__(self):
        if getattr(self, "h", None) and self.lib is not None:
            self.lib.souffle_graph_destroy(self.h)
            self.h = None

    def _out(self, f, *args):
        o = C.c_int32()
        check(f(self.h, *args, C.byref(o)))
        return o.value

    def placeholder(self, shape, dtype=F32, const=True):
        return self._out(self.lib.souffle_placeholder, len(shape), _i64(shape), dtype, 1 if const else 0)

    def matmul(self, a, b, trans_b=True, prec=F32):
        return self._out(self.lib.souffle_matmul, a, b, 1 if trans_b else 0, prec)

    def ew(self, fn, *ins, scalar=0.0):
        return self._out(self.lib.souffle_elementwise, EW[fn], len(ins), _i32(ins), float(scalar))

    def reduce(self, fn, x, axis, keepdim=True):
        return self._out(self.lib.souffle_reduce, RED[fn], x, axis, 1 if keepdim else 0)

    def reshape(self, x, shape):
        return self._out(self.lib.souffle_reshape, x, len(shape), _i64(shape))

    def permute(self, x, perm):
        return self._out(self.lib.souffle_permute, x, _i32(perm))

    def slice(self, x, begin, end, stride):
        return self._out(self.lib.souffle_slice, x, _i64(begin), _i64(end), _i64(stride))

    def roll(self, x, shifts):
        return self._out(self.lib.souffle_roll, x, _i64(shifts))

    def mark_output(self, t):
        check(self.lib.souffle_mark_output(self.h, t))
        if t not in self.outputs:
            self.outputs.append(t)

    def num_nodes(self):
        n = C.c_int32()
        check(self.lib.souffle_graph_num_nodes(self.h, C.byref(n)))
        return n.value

    def node(self, t):
        op, nd, dt = C.c_int32(), C.c_int32(), C.c_int32()
        shp = (C.c_int64 * 8)()
        check(self.lib.souffle_graph_node(self.h, t, C.byref(op), C.byref(nd), shp, C.byref(dt)))
        return op.value, tuple(shp[:nd.value]), dt.value

    def set_te_resources(self, te, grid, smem, regs=0, threads=0):
        check(self.lib.souffle_set_te_resources(self.h, te, grid, smem, regs, threads))

    def partition(self, dev=None, flags=0):
        return Plan(self, dev or device_b200(), flags)


def device_b200():
    d = DeviceDesc()
    check(load().souffle_device_b200(C.byref(d)))
    return d


def device_query(dev=0):
    d = DeviceDesc()
    check(load().souffle_device_query(dev, C.byref(d)))
    return d


def paper_device(capacity_bytes):
    """The paper's analytical rule (§5.4): max_grid * max_smem <= C."""
    d = DeviceDesc()
    d.rule = 1
    d.capacity_C = capacity_bytes
    return d


class Plan:
    """souffle_partition result: introspection + execution (souffle_bind / souffle_run)."""

    def __init__(self, graph, dev, flags=0):
        self.lib = graph.lib
        h = C.c_void_p()
        check(self.lib.souffle_partition(graph.h, C.byref(dev), flags, C.byref(h)))
        self.h = h
        self.flags = flags

    def __del__(self):
        if getattr(self, "h", None) and self.lib is not None:
            self.lib.souffle_plan_destroy(self.h)
            self.h = None

    def _int(self, f):
        n = C.c_int32()
        check(f(self.h, C.byref(n)))
        return n.value

    def num_nodes(self):
        return self._int(self.lib.souffle_plan_num_nodes)

    def num_tes(self):
        return self._int(self.lib.souffle_plan_num_tes)

    def num_subprograms(self):
        return self._int(self.lib.souffle_plan_num_subprograms)

    def assignment(self):
        a = (C.c_int32 * self.num_nodes())()
        check(self.lib.souffle_plan_assignment(self.h, a))
        return list(a)

    def bfs_order(self):
        a = (C.c_int32 * max(1, self.num_tes()))()
        check(self.lib.souffle_plan_bfs_order(self.h, a))
        return list(a)[: self.num_tes()]

    def te_info(self, t):
        v = [C.c_int32(), C.c_int32(), C.c_int64(), C.c_int64(), C.c_int64(), C.c_int64(), C.c_int32(), C.c_int32()]
        check(self.lib.souffle_plan_te_info(self.h, t, *[C.byref(x) for x in v]))
        k = ["dep", "ci", "ops", "accesses", "grid", "smem", "regs", "threads"]
        return dict(zip(k, [x.value for x in v]))

    def reuse_set(self, t, cap=4096):
        buf = (C.c_int32 * cap)()
        n, kind = C.c_int32(), C.c_int32()
        check(self.lib.souffle_plan_reuse_set(self.h, t, buf, cap, C.byref(n), C.byref(kind)))
        return list(buf[: min(n.value, cap)]), kind.value

    def index_map(self, t, s, numel):
        buf = (C.c_int64 * numel)()
        check(self.lib.souffle_plan_index_map(self.h, t, s, buf))
        return list(buf)

    def hgroup(self, t):
        lv, g, k = C.c_int32(), C.c_int32(), C.c_int32()
        check(self.lib.souffle_plan_hgroup(self.h, t, C.byref(lv), C.byref(g), C.byref(k)))
        return lv.value, g.value, k.value

    def exec_info(self):
        a, b, c = C.c_int32(), C.c_int32(), C.c_int32()
        check(self.lib.souffle_plan_exec_info(self.h, C.byref(a), C.byref(b), C.byref(c)))
        return dict(launches=a.value, stages=b.value, barriers=c.value)

    def describe(self):
        s = C.c_char_p()
        check(self.lib.souffle_plan_describe(self.h, C.byref(s)))
        return s.value.decode()

    def workspace_bytes(self):
        n = C.c_size_t()
        check(self.lib.souffle_plan_workspace_bytes(self.h, C.byref(n)))
        return n.value

    def bind(self, t, ptr):
        check(self.lib.souffle_bind(self.h, t, C.c_void_p(int(ptr))))

    def workspace_init(self, ws_ptr, stream=0):
        check(self.lib.souffle_workspace_init(self.h, C.c_void_p(int(ws_ptr)), C.c_void_p(int(stream))))

    def set_profiling(self, on=True):
        check(self.lib.souffle_plan_set_profiling(self.h, 1 if on else 0))

    def read_profile(self, ws_ptr):
        n = self.exec_info()["stages"]
        buf = (C.c_double * max(1, n))()
        got = C.c_int32()
        check(self.lib.souffle_plan_read_profile(self.h, C.c_void_p(int(ws_ptr)), buf, n, C.byref(got)))
        return list(buf[: got.value])

    def run(self, ws_ptr, stream=0):
        check(self.lib.souffle_run(self.h, C.c_void_p(int(ws_ptr)), C.c_void_p(int(stream))))


def _add_raw_profile():
    def read_profile_raw(self, ws_ptr):
        n = self.exec_info()["stages"]
        cap = 9 * n + 1 + 4 * 160 * n   # stage starts, 8 marks per stage, per-CTA marks
        buf = (C.c_uint64 * cap)()
        got = C.c_int32()
        check(self.lib.souffle_plan_read_profile_raw(self.h, C.c_void_p(int(ws_ptr)), buf, cap, C.byref(got)))
        starts = list(buf[: n + 1])
        marks = [list(buf[n + 1 + 8 * s: n + 1 + 8 * s + 8]) for s in range(n)]
        return starts, marks
    Plan.read_profile_raw = read_profile_raw


_SIGS["souffle_plan_read_profile_raw"] = [C.c_void_p, C.c_void_p, C.POINTER(C.c_uint64), C.c_int32,
                                          C.POINTER(C.c_int32)]
_SIGS["souffle_plan_debug_region"] = [C.c_void_p, C.c_char_p, C.POINTER(C.c_int64), C.POINTER(C.c_int64)]


def _debug_region(self, name):
    """(byte offset, bytes) of a named BERT-kernel workspace buffer (stage-isolation tests)."""
    o, b = C.c_int64(), C.c_int64()
    check(self.lib.souffle_plan_debug_region(self.h, name.encode(), C.byref(o), C.byref(b)))
    return o.value, b.value


Plan.debug_region = _debug_region
EXPORTS = sorted(list(_SIGS) + ["souffle_last_error", "souffle_version"])
_add_raw_profile()
