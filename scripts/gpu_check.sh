mkdir -p gpurun_out; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider 2>&1 | tail -40 > gpurun_out/pytest_gpu.txt
timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench1.txt 2>&1
tail -3 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; tail -3 gpurun_out/bench1.txt
