#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
# launch ids of one run (after the first): 0 bias, 1 im2col, 2 embed gemm, 3 LN, then blocks of 7 (+2 per merge)
# stage-3 first block starts at 4 + 14 + 2 + 14 + 2 = 36: LN1 36, QKV 37, ATTN 38, PROJ 39, LN2 40, FC1 41, FC2 42
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sw_gemm -s 21 -c 1 -o gpurun_out/prof_swin_fc1 python tools/run_swin_once.py 64 1 > gpurun_out/ncu_swin_fc1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sw_gemm -s 22 -c 1 -o gpurun_out/prof_swin_fc2 python tools/run_swin_once.py 64 1 > gpurun_out/ncu_swin_fc2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bert_kernel -s 1 -c 1 -o gpurun_out/prof_bert2 python tools/run_once.py bert_base 0 0 2 > gpurun_out/ncu_bert2.log 2>&1
echo done
