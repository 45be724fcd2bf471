"""Device time per inference of the small models (MMoE, LSTM) from a CUDA-graph replay of 100
back-to-back inferences (no per-launch CPU submission in the timed region), plus an empty kernel
replayed the same way as the per-launch floor.  Prints one JSON object.
usage: python tools/graph_timing.py"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402


def graph_us(fn, reps=100, trials=7, sess=None):
    s = torch.cuda.Stream()
    if sess is not None:      # the library launches on the session's stream: capture on that one
        sess.stream = s
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(reps):
            fn()
    g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(trials):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b) * 1e3 / reps)
    return statistics.median(ts)


def main():
    import bench
    out = {}
    mplan, msess = bench.build_mmoe(0)
    out["mmoe_us_per_inference_graph100"] = graph_us(msess.run, sess=msess)
    lplan, lsess, lcfg = bench.build_lstm(0)
    out["lstm_us_per_inference_graph20"] = graph_us(lsess.run, reps=20, sess=lsess)
    x = torch.zeros(1, device="cuda")
    out["empty_kernel_us_graph100"] = graph_us(lambda: x.add_(1))
    print(json.dumps(out))


if __name__ == "__main__":
    main()
