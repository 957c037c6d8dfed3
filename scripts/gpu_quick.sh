mkdir -p gpurun_out; rm -f gpurun_out/quick.txt
for c in "C2 fp32" "C2 mixed" "C2 fp16" "C1 fp32" "C1 mixed" "C1 fp64" "X64_32768_256 fp32" "X64_32768_256 mixed"; do timeout 300 python scripts/prof_one.py $c 1 >> gpurun_out/quick.txt 2>&1; done
cat gpurun_out/quick.txt
