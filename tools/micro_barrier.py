"""Microbenchmark: cost per dependent stage (grid barrier + a tiny elementwise stage).

A chain of n `neg` TEs with vertical fusion disabled lowers to n EW stages separated by n-1 grid
barriers in one persistent launch.  Reports device time per stage for several tensor sizes."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402


def chain(rows, cols, n, flags):
    g = L.Graph()
    x = g.placeholder((rows, cols), L.F32, const=False)
    h = x
    for _ in range(n):
        h = g.ew("neg", h)
    g.mark_output(h)
    plan = g.partition(L.device_query(0), flags)
    s = session(g, plan, {x: np.ones((rows, cols), np.float32)}, [h])
    for _ in range(3):
        s.run()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(10):
        s.run()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / 10 * 1e3, plan.exec_info()


if __name__ == "__main__":
    n = 64
    for rows, cols in ((1, 8), (128, 768), (1024, 768)):
        t, info = chain(rows, cols, n, L.FLAG_NO_VERTICAL)
        print(f"[{rows}x{cols}] {n} stages: {t:8.1f} us total, {t / n:6.2f} us/stage  {info}")
    t, info = chain(128, 768, n, L.FLAG_NO_VERTICAL | L.FLAG_NO_GLOBAL_SYNC)
    print(f"[128x768] one launch per stage: {t / n:6.2f} us/stage  {info}")
    t, info = chain(128, 768, n, 0)
    print(f"[128x768] vertically fused: {t:8.1f} us total  {info}")
