# half-precision kernel check: GPU tests of the half modes + timings
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf -x -p no:cacheprovider -k "half or c3 or smoke" > gpurun_out/pytest_half.txt 2>&1
tail -15 gpurun_out/pytest_half.txt
for c in "C2 mixed" "C2 fp16" "C2 fp16c" "C1 mixed" "C3 mixed"; do timeout 600 python scripts/prof_one.py $c 2 >> gpurun_out/prof_half.txt 2>&1; done
cat gpurun_out/prof_half.txt
