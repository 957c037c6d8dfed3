# FP32 accuracy / speed check (full-grid err/tol vs the FP64 path, per re-seed interval) + all GPU tests
mkdir -p gpurun_out; o=gpurun_out/fp32acc.txt; rm -f $o
timeout 300 python scripts/fp32_err_map.py X64_32768_256 0 512 256 >> $o 2>&1
timeout 600 python scripts/fp32_err_map.py C3 0 512 >> $o 2>&1
timeout 300 python scripts/fp32_err_map.py C2 0 >> $o 2>&1
timeout 300 python scripts/fp32_err_map.py X256_8192_512 0 512 256 >> $o 2>&1
for c in "C2 fp32" "X64_32768_256 fp32"; do timeout 300 python scripts/prof_one.py $c 2 >> $o 2>&1; done
timeout 1500 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1
timeout 1500 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
grep -v "^  k=" $o; tail -3 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt; cut -c1-300 gpurun_out/bench_default.json
