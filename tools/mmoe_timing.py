import sys, os, statistics
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import torch, bench
plan, sess = bench.build_mmoe(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
st = torch.cuda.current_stream()
cold = bench.time_steps(sess, 50, 5, flush, st)
warm = []
for i in range(60):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); sess.run(); b.record(); b.synchronize()
    if i >= 10: warm.append(a.elapsed_time(b) * 1e3)
x = torch.zeros(1, device="cuda")
triv = []
for i in range(60):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); x.add_(1); b.record(); b.synchronize()
    if i >= 10: triv.append(a.elapsed_time(b) * 1e3)
print("mmoe cold", statistics.median(cold) * 1e3, "warm", statistics.median(warm), "trivial kernel", statistics.median(triv))
