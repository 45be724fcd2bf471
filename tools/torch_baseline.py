"""Context baseline (not part of the product path): the same BERT-base b1 s128 graph run op by op with
PyTorch on the same weights -- cuBLAS bf16 GEMMs, fused SDPA attention, fp32 LayerNorm, erf GELU --
captured in a CUDA graph, L2 flushed before every replay (outside the events), median latency.
usage: python tools/torch_baseline.py"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import torch.nn.functional as F  # noqa: E402

import synth  # noqa: E402

def measure(dev="cuda", replays=50, eager_runs=15):
    """Median latencies (us) of the op-by-op torch BERT-base: CUDA-graph replay and eager."""
    cfg = synth.BERT_BASE
    S, H, nh, FF = cfg["seq"], cfg["hidden"], cfg["heads"], cfg["ffn"]
    d = H // nh
    x0 = torch.from_numpy(synth.bert_input(cfg)).to(dev)
    layers = []
    for wl in synth.bert_weights(cfg):
        t = {k: torch.from_numpy(v).to(dev) for k, v in wl.items()}
        for k in ("Wq", "Wk", "Wv", "Wo", "W1", "W2"):
            t[k] = t[k].to(torch.bfloat16)
        t["Wqkv"] = torch.cat([t["Wq"], t["Wk"], t["Wv"]], 0)
        t["bqkv"] = torch.cat([t["bq"], t["bk"], t["bv"]], 0)
        layers.append(t)


    def forward(x):
        for t in layers:
            qkv = F.linear(x.to(torch.bfloat16), t["Wqkv"]).float() + t["bqkv"]
            q, k, v = qkv.view(S, 3, nh, d).permute(1, 2, 0, 3).to(torch.bfloat16)
            ctx = F.scaled_dot_product_attention(q.unsqueeze(0), k.unsqueeze(0), v.unsqueeze(0))[0]
            ctx = ctx.permute(1, 0, 2).reshape(S, H)
            a = F.linear(ctx, t["Wo"]).float() + t["bo"] + x
            l1 = F.layer_norm(a, (H,), t["g1"], t["be1"], eps=1e-12)
            h = F.gelu(F.linear(l1.to(torch.bfloat16), t["W1"]).float() + t["c1"])
            o = F.linear(h.to(torch.bfloat16), t["W2"]).float() + t["c2"] + l1
            x = F.layer_norm(o, (H,), t["g2"], t["be2"], eps=1e-12)
        return x


    xs = x0.clone()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            y = forward(xs)
    torch.cuda.current_stream().wait_stream(s)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        y = forward(xs)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    ts = []
    for i in range(replays + 10):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        b.synchronize()
        if i >= 10:
            ts.append(a.elapsed_time(b) * 1e3)
    eager = []
    for i in range(eager_runs + 5):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        forward(xs)
        b.record()
        b.synchronize()
        if i >= 5:
            eager.append(a.elapsed_time(b) * 1e3)
    return {"workload": "BERT-base b1 s128, torch op-by-op (cuBLAS bf16 GEMMs, SDPA, fp32 LN)",
            "cuda_graph_latency_us": statistics.median(ts), "eager_latency_us": statistics.median(eager),
            "torch": torch.__version__}


if __name__ == "__main__":
    print(json.dumps(measure()))
