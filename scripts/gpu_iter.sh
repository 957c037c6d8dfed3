# quick iteration: GPU parity tests + main-kernel timings of the C2 modes (+ EXTRA_CASES="name:prec ...")
mkdir -p gpurun_out; rm -f gpurun_out/iter.txt
timeout 1500 python -m pytest tests -m gpu -x -q -rf -p no:cacheprovider ${PYTEST_K} > gpurun_out/pytest_gpu.txt 2>&1
tail -3 gpurun_out/pytest_gpu.txt >> gpurun_out/iter.txt
for c in ${CASES:-C2:fp32 C2:fp64 C2:mixed C2:fp16 C2:fp16c} ${EXTRA_CASES}; do timeout 600 python scripts/prof_one.py ${c%%:*} ${c##*:} 2 >> gpurun_out/iter.txt 2>&1; done
cat gpurun_out/iter.txt
