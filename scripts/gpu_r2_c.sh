mkdir -p gpurun_out/sanitize
CS=/usr/local/cuda/bin/compute-sanitizer
for c in "fp32 4 self" "fp32 16 self" "fp64 64 self" "fp64 64 ab" "mixed 8 self" "mixed 16 ab" "mixed 64 self" "fp16 64 ab" "fp16c 16 self" "fp32 64 self" "fp16 256 self" "fp64 256 self"; do
  tag=$(echo $c | tr ' ' '_')
  timeout 900 $CS --tool racecheck --print-limit 20 python scripts/sanitize_case.py $c 160 16 > gpurun_out/sanitize/racecheck2_$tag.txt 2>&1
  echo "racecheck $c rc=$? $(grep -E 'RACECHECK SUMMARY' gpurun_out/sanitize/racecheck2_$tag.txt | tail -1)"
done | tee gpurun_out/sanitize/summary2.txt
timeout 1800 python -m pytest tests -m gpu -q -rf -p no:cacheprovider -x > gpurun_out/pytest_gpu.txt 2>&1; tail -3 gpurun_out/pytest_gpu.txt
timeout 1200 python scripts/embedded_recall.py > gpurun_out/embedded_recall.txt 2>&1; cp profiles/r2_embedded_recall.json gpurun_out/ 2>/dev/null; cat gpurun_out/embedded_recall.txt | tail -25
