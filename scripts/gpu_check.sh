mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -q -rf -s -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1
for c in "C2 fp32" "C2 fp64" "C2 mixed" "C2 fp16" "C1 fp32" "C1 fp64" "C3 fp32" "C3 mixed"; do timeout 600 python scripts/prof_one.py $c 2 >> gpurun_out/prof_one.txt 2>&1; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/prof_c2_fp32_v10 python scripts/prof_one.py C2 fp32 2 > gpurun_out/ncu_log.txt 2>&1
tail -5 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt gpurun_out/prof_one.txt; tail -3 gpurun_out/ncu_log.txt
