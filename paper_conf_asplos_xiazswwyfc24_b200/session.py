"""Device-memory plumbing around a plan (PyTorch owns device memory and streams).

A Session allocates the bound tensors and the workspace with torch, binds them through the C ABI
(souffle_bind / souffle_workspace_init) and runs the plan with souffle_run on a torch stream.
No compute happens here: every TE runs in libsouffle's sm_100a kernels.  There is no CPU fallback:
constructing a Session without a CUDA device raises.
"""
from __future__ import annotations

import numpy as np
import torch

from . import _lib as L


def _torch_dtype(dt):
    return torch.bfloat16 if dt == L.BF16 else torch.float32


def to_device(arr, dtype, device):
    """Copy stored values (float32 arrays exactly representable in dtype) to a device tensor."""
    t = torch.from_numpy(np.ascontiguousarray(arr, dtype=np.float32))
    return t.to(device=device, dtype=_torch_dtype(dtype))


class Session:
    def __init__(self, graph: L.Graph, plan: L.Plan, feed: dict, device="cuda:0", stream=None):
        if not torch.cuda.is_available():
            raise RuntimeError("souffle Session needs a CUDA (sm_100a) device; there is no CPU fallback")
        self.graph, self.plan = graph, plan
        self.device = torch.device(device)
        self.stream = stream or torch.cuda.current_stream(self.device)
        self.inputs = {}
        for t, arr in feed.items():
            op, shape, dt = graph.node(t)
            assert op == L.OP_PLACEHOLDER, t
            x = to_device(np.asarray(arr).reshape(shape), dt, self.device)
            self.inputs[t] = x
            plan.bind(t, x.data_ptr())
        self.outputs = {}
        for t in self.output_ids():
            _, shape, _ = graph.node(t)
            y = torch.zeros(shape, dtype=torch.float32, device=self.device)
            self.outputs[t] = y
            plan.bind(t, y.data_ptr())
        self.ws = torch.zeros(plan.workspace_bytes(), dtype=torch.uint8, device=self.device)
        plan.workspace_init(self.ws.data_ptr(), self.stream.cuda_stream)

    def output_ids(self):
        return self._outs

    def run(self):
        self.plan.run(self.ws.data_ptr(), self.stream.cuda_stream)

    def result(self, t):
        torch.cuda.synchronize(self.device)
        return self.outputs[t].double().cpu().numpy()


def session(graph, plan, feed, outputs=None, **kw):
    """Bind every marked output of `graph` (plus any extra ids in `outputs`)."""
    s = Session.__new__(Session)
    outs = list(graph.outputs)
    for o in outputs or []:
        if o not in outs:
            outs.append(o)
    s._outs = outs
    Session.__init__(s, graph, plan, feed, **kw)
    return s
