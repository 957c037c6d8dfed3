# GPU tests + ncu captures: full --set full of the main kernel on named cases, launch list of the bench
mkdir -p gpurun_out
[ -z "$NOTEST" ] && timeout 2400 python -m pytest tests -m gpu -q -rf -s -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; tail -3 gpurun_out/pytest_gpu.txt
for pc in ${NCU_CASES}; do
  tag=$(echo $pc | tr ':' '_')
  timeout 1500 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s ${NCU_SKIP:-1} -c 1 -o gpurun_out/full_$tag python scripts/prof_one.py ${pc%%:*} ${pc##*:} 1 > gpurun_out/ncu_$tag.log 2>&1
  tail -1 gpurun_out/ncu_$tag.log
done
[ -n "$LAUNCHES" ] && timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-per-precision --no-per-config --no-context > gpurun_out/bench_under_ncu.txt 2>&1; tail -2 gpurun_out/bench_under_ncu.txt
