mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt; lscpu | grep "Model name" >> gpurun_out/nproc.txt
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-per-precision > gpurun_out/bench_under_ncu.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/prof_r1_c2_fp32 python scripts/prof_one.py C2 fp32 2 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/prof_r1_c2_fp64 python scripts/prof_one.py C2 fp64 2 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/prof_r1_c2_mixed python scripts/prof_one.py C2 mixed 2 > /dev/null 2>&1
cat gpurun_out/bench_default.json gpurun_out/bench_reference.json; tail -3 gpurun_out/bench_default.err
