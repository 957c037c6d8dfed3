mkdir -p gpurun_out; rm -f gpurun_out/prof_one.txt
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1500 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1
for c in "C2 fp32" "C2 fp64" "C2 mixed" "C2 fp16" "C2 fp16c" "C1 fp32" "C1 fp64" "C1 mixed" "C3 fp32" "C3 mixed"; do timeout 600 python scripts/prof_one.py $c 2 >> gpurun_out/prof_one.txt 2>&1; done
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
tail -5 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt gpurun_out/prof_one.txt gpurun_out/bench_default.json
