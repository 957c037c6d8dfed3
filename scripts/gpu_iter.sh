# one iteration: GPU parity tests, timings of a case list, optional ncu of one case
mkdir -p gpurun_out; rm -f gpurun_out/iter.txt
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
tail -3 gpurun_out/pytest_gpu.txt >> gpurun_out/iter.txt
while read -r c; do [ -n "$c" ] && timeout 600 python scripts/prof_one.py $c 1 >> gpurun_out/iter.txt 2>&1; done <<< "$CASES"
if [ -n "$NCU" ]; then
  tag=$(echo $NCU | tr ' ' '_')
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/ncu_$tag python scripts/prof_one.py $NCU 1 > gpurun_out/ncu_$tag.log 2>&1
  tail -1 gpurun_out/ncu_$tag.log >> gpurun_out/iter.txt
fi
cat gpurun_out/iter.txt
