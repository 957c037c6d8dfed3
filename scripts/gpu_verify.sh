mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1500 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1
timeout 1500 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
tail -3 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; cut -c1-600 gpurun_out/bench_default.json; tail -3 gpurun_out/bench_default.err
