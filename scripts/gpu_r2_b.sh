mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_stages.py -q -rf -p no:cacheprovider > gpurun_out/pytest_stages.txt 2>&1; tail -3 gpurun_out/pytest_stages.txt
MP_PARITY_NO_COND=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -p no:cacheprovider -k "random_shapes and fp32 or reseed and fp32" > gpurun_out/pytest_nocond.txt 2>&1; tail -8 gpurun_out/pytest_nocond.txt
bash scripts/gpu_sanitize.sh
