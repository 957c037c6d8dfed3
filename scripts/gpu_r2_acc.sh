# round 2: FP32 compensated recurrence -- full-grid err/tol vs the FP64 path, timings, GPU tests
mkdir -p gpurun_out; o=gpurun_out/fp32acc.txt; rm -f $o
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
for c in "C2 fp32" "X64_32768_256 fp32" "X256_8192_512 fp32" "C3 fp32"; do timeout 600 python scripts/prof_one.py $c 2 >> gpurun_out/prof_one.txt 2>&1; done
timeout 300 python scripts/fp32_err_map.py C2 0 >> $o 2>&1
timeout 300 python scripts/fp32_err_map.py X64_32768_256 0 >> $o 2>&1
timeout 300 python scripts/fp32_err_map.py X256_8192_512 0 >> $o 2>&1
timeout 600 python scripts/fp32_err_map.py X256_32768_512 0 >> $o 2>&1
timeout 900 python scripts/fp32_err_map.py C3 0 >> $o 2>&1
timeout 1500 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
grep -v "^  k=" $o; tail -5 gpurun_out/pytest_gpu.txt; cat gpurun_out/prof_one.txt
