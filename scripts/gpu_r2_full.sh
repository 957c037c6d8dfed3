# round-2 full measurement batch: GPU tests, smoke, bench line (C3) + reference arm, launch list of
# the bench, one ncu --set full capture per NCU_CASES entry ("<config>:<precision>")
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1
[ -z "$NOTEST" ] && timeout 2400 python -m pytest tests -m gpu -q -rf -s -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; tail -2 gpurun_out/pytest_gpu.txt
[ -z "$NOTEST" ] && timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
[ -z "$NOBENCH" ] && timeout 1800 python bench.py $BENCH_ARGS > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -2 gpurun_out/bench_default.err; cut -c1-400 gpurun_out/bench_default.json
[ -n "$REF" ] && timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; cut -c1-300 gpurun_out/bench_reference.json 2>/dev/null
[ -n "$LAUNCHES" ] && timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-per-precision --no-per-config --no-context > gpurun_out/bench_under_ncu.txt 2>&1; tail -1 gpurun_out/bench_under_ncu.txt
for pc in ${NCU_CASES}; do
  tag=$(echo $pc | tr ':' '_')
  timeout 1500 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s ${NCU_SKIP:-1} -c 1 -o gpurun_out/full_$tag python scripts/prof_one.py ${pc%%:*} ${pc##*:} 1 > gpurun_out/ncu_$tag.log 2>&1
  tail -1 gpurun_out/ncu_$tag.log
done
exit 0
