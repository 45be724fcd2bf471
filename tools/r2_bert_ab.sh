#!/bin/bash
# BERT timing A/B of the arrival variants (dbg bits), plus parity
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
for v in 0 1048576 2097152 3145728; do
  SOUFFLE_BERT_DBG_SKIP=$v timeout 300 python tools/sweep_bert.py "" > gpurun_out/ab_$v.txt 2>&1
done
timeout 600 python -m pytest tests/test_gpu_bert_stages.py tests/test_gpu_parity.py -q -x -m gpu -k "bert or stage or layernorm or bias" > gpurun_out/pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_bert.txt
echo done
