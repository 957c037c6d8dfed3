# round-2 measurement batch: GPU tests, smoke, half-mode bounds, bench line (C3), reference arm
mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt; lscpu | grep "Model name" >> gpurun_out/nproc.txt
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 2400 python -m pytest tests -m gpu -q -rf -s -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
tail -5 gpurun_out/pytest_gpu.txt
timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1; tail -3 gpurun_out/smoke.txt
[ -n "$HALF" ] && timeout 1200 python scripts/half_bounds.py C1 C2 C3 > gpurun_out/half_bounds.txt 2>&1 && cp profiles/r2_half_bounds.json gpurun_out/
timeout 1800 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
tail -3 gpurun_out/bench_default.err; cut -c1-600 gpurun_out/bench_default.json
[ -n "$REF" ] && timeout 1200 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; cut -c1-400 gpurun_out/bench_reference.json
