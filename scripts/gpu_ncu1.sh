mkdir -p gpurun_out
for c in "$@"; do
  tag=$(echo $c | tr ' ' '_')
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/ncu_$tag python scripts/prof_one.py $c 1 > gpurun_out/ncu_$tag.log 2>&1
  tail -2 gpurun_out/ncu_$tag.log
done
