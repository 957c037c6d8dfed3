mkdir -p gpurun_out/sanitize
CS=/usr/local/cuda/bin/compute-sanitizer
for c in "mixed 8 self" "mixed 16 ab" "mixed 64 self" "fp16 64 ab" "fp16c 16 self" "fp16 256 self"; do
  tag=$(echo $c | tr ' ' '_')
  timeout 900 $CS --tool racecheck --print-limit 20 python scripts/sanitize_case.py $c 160 16 > gpurun_out/sanitize/racecheck4_$tag.txt 2>&1
  echo "racecheck $c rc=$? $(grep -E 'RACECHECK SUMMARY' gpurun_out/sanitize/racecheck4_$tag.txt | tail -1)"
done | tee gpurun_out/sanitize/summary4.txt
timeout 900 python -m pytest tests -m gpu -q -rf -p no:cacheprovider -k "half" > gpurun_out/pytest_half.txt 2>&1; tail -2 gpurun_out/pytest_half.txt
VARIANTS="exp_pre exp_base exp_wm4" CASES="C2:mixed C2:fp16 C2:fp32 X64_32768_256:mixed X256_8192_512:mixed X256_8192_512:fp16" bash scripts/gpu_variants.sh
