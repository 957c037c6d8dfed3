mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rf -s -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
timeout 900 python scripts/accuracy_study.py > gpurun_out/accuracy.txt 2>&1
cp profiles/r1_accuracy.json gpurun_out/ 2>/dev/null
tail -3 gpurun_out/pytest_gpu.txt; cat gpurun_out/accuracy.txt | head -70
