mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-per-precision --no-per-config > gpurun_out/bench_under_ncu.txt 2>&1
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
tail -2 gpurun_out/bench_under_ncu.txt; wc -l gpurun_out/launches.csv; cut -c1-300 gpurun_out/bench_reference.json
