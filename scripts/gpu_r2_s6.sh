# sign-split merge: FP32 stage + parity tests, then C3 / X64 timing vs the lane-dependent merge
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1; tail -1 gpurun_out/build.txt
timeout 1200 python -m pytest tests/test_gpu_stages.py tests/test_gpu_parity.py -q -rf -p no:cacheprovider -k "fp32 or sort or stage" > gpurun_out/pytest_sign.txt 2>&1; tail -3 gpurun_out/pytest_sign.txt
CASES="C3:fp32 X64_32768_256:fp32" VARIANTS="main exp_nosign" bash scripts/gpu_r2_s4.sh
exit 0
