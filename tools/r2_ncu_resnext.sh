#!/bin/bash
# ncu --set full of the ResNeXt pattern kernel on R5 (14x14, 1024 channels, the block repeated 22x)
mkdir -p gpurun_out
cat > /tmp/rx_once.py <<'PY'
import os, sys
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import torch, synth
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L, models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session
cfg = synth.RESNEXT_CONFIGS[5]
p = {**synth.resnext_params(cfg), **synth.resnext_masks(cfg)}
g, names, gx, gy = M.resnext(cfg)
plan = g.partition(L.device_query(0))
s = session(g, plan, {names[k]: v for k, v in p.items()} | {gx: synth.resnext_input(cfg)}, [gy])
for _ in range(3):
    s.run()
torch.cuda.synchronize()
print("ok")
PY
timeout 900 ncu --set full --import-source on --clock-control none -k regex:resnext_kernel -s 2 -c 1 -o gpurun_out/ncu_resnext python /tmp/rx_once.py > gpurun_out/ncu_resnext.log 2>&1
echo done
