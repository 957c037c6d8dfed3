# round 2: new large-d FP32 kernel (mp_diag_ctab) -- correctness, accuracy and variant timings
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 600 python -m pytest tests -m gpu -q -x -rf -p no:cacheprovider -k "shapes or long or c3 or band or c1" > gpurun_out/pytest_gpu.txt 2>&1
tail -15 gpurun_out/pytest_gpu.txt
timeout 300 python scripts/fp32_err_map.py X64_32768_256 0 > gpurun_out/fp32acc.txt 2>&1
timeout 300 python scripts/fp32_err_map.py X256_8192_512 0 >> gpurun_out/fp32acc.txt 2>&1
grep -v "^  k=" gpurun_out/fp32acc.txt
VARIANTS="exp_base exp_m2 exp_dl32 exp_old exp_f8" CASES="X64_32768_256:fp32 X256_8192_512:fp32 X128_16384_256:fp32 C2:fp32" bash scripts/gpu_variants.sh
