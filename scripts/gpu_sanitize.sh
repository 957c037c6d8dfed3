# compute-sanitizer over every kernel family (warp / block-cooperative; FP32, FP64, half; self / AB)
mkdir -p gpurun_out/sanitize; rm -f gpurun_out/sanitize/*
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  for c in "fp32 4 self" "fp32 16 self" "fp32 16 ab" "fp32 64 self" "fp32 64 ab" "fp32 256 self" \
           "fp64 4 self" "fp64 16 self" "fp64 64 self" "fp64 64 ab" \
           "mixed 8 self" "mixed 16 ab" "mixed 64 self" "fp16 64 ab" "fp16c 16 self"; do
    tag=$(echo $c | tr ' ' '_')
    n=300; [ $tool = racecheck ] && n=160
    timeout 900 $CS --tool $tool --print-limit 20 python scripts/sanitize_case.py $c $n 16 > gpurun_out/sanitize/${tool}_$tag.txt 2>&1
    echo "$tool $c rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' gpurun_out/sanitize/${tool}_$tag.txt | tail -1)"
  done
done | tee gpurun_out/sanitize/summary.txt
