mkdir -p gpurun_out
for d in 0 32768 65536 98304; do
  echo "== DBG $d" >> gpurun_out/prof_dbg.txt
  SOUFFLE_BERT_DBG_SKIP=$d timeout 100 python tools/profile_bert.py 2 >> gpurun_out/prof_dbg.txt 2>&1
done
