# round-end style measurement: GPU tests, bench line, reference arm, ncu launch list,
# ncu --set full captures of the hot kernels, accuracy study
mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt; lscpu | grep "Model name" >> gpurun_out/nproc.txt
timeout 1500 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1
timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1
timeout 1500 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-per-precision --no-per-config > gpurun_out/bench_under_ncu.txt 2>&1
for pc in ${NCU_CASES:-C2:fp32 C2:fp64 C2:mixed C2:fp16 X64_32768_256:mixed X64_32768_256:fp32 X64_32768_256:fp64}; do
  tag=$(echo $pc | tr ':' '_')
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/full_$tag python scripts/prof_one.py ${pc%%:*} ${pc##*:} 1 > /dev/null 2>&1
done
timeout 1200 python scripts/accuracy_study.py > gpurun_out/accuracy.txt 2>&1; cp profiles/r1_accuracy.json gpurun_out/ 2>/dev/null
tail -3 gpurun_out/pytest_gpu.txt; cat gpurun_out/smoke.txt gpurun_out/bench_default.json gpurun_out/bench_reference.json; tail -3 gpurun_out/bench_default.err; tail -5 gpurun_out/accuracy.txt
