# round-2 final measurement batch: GPU tests, smoke, bench line (C3) + reference arm, launch list,
# ncu --set full of the tensor-core seed GEMM (X64 Mixed, seed_mode tc)
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1; tail -1 gpurun_out/build.txt
[ -z "$NOTEST" ] && timeout 2400 python -m pytest tests -m gpu -q -rf -s -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; tail -2 gpurun_out/pytest_gpu.txt
[ -z "$NOTEST" ] && timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
timeout 1800 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -2 gpurun_out/bench_default.err; cut -c1-300 gpurun_out/bench_default.json
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; cut -c1-200 gpurun_out/bench_reference.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-per-precision --no-per-config --no-context --no-stream > gpurun_out/bench_under_ncu.txt 2>&1; tail -1 gpurun_out/bench_under_ncu.txt | cut -c1-200
echo skip-ncu
exit 0
