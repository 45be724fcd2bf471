#!/bin/bash
# round-2 final evidence: full GPU suite (errors logged), the default bench line, the bench's ncu
# launch list, one ncu --set full capture of the BERT kernel, BERT stage timeline, Swin traces
mkdir -p gpurun_out
rm -f gpurun_out/parity_errors.jsonl
nvidia-smi > gpurun_out/r02_nvsmi.txt 2>&1
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/r02_pytest_gpu.txt 2>&1
echo "rc=$?" >> gpurun_out/r02_pytest_gpu.txt
timeout 600 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/r02_smoke.txt 2>&1
echo "rc=$?" >> gpurun_out/r02_smoke.txt
timeout 1500 python bench.py > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-v0 --no-models > gpurun_out/r02_ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bert_kernel -s 1 -c 1 -o gpurun_out/r02_prof_bert python tools/run_once.py bert_base 0 0 2 > gpurun_out/r02_ncu_full.log 2>&1
timeout 300 python tools/profile_bert.py 12 > gpurun_out/r02_timeline.txt 2>&1
timeout 600 ncu --set full --clock-control none -k regex:mmoe_cluster_kernel -s 3 -c 1 -o gpurun_out/r02_prof_mmoe python tools/run_model_once.py mmoe 6 > gpurun_out/r02_ncu_mmoe.log 2>&1
timeout 600 python tools/profile_resnext.py > gpurun_out/r02_resnext_phases.txt 2>&1
for b in 1 8 64; do timeout 300 python tools/swin_trace.py $b > gpurun_out/r02_swin_trace_b$b.txt 2>&1; done
echo done
