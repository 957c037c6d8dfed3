# session-2 checks: new GPU tests (streaming, tensor-core seeds, FP16CK), quick bench, C3 Mixed
# direct vs tensor-core seeds timing
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1; tail -1 gpurun_out/build.txt
timeout 900 python -m pytest tests/test_gpu_seeds_tc.py -x -q -rf -s -p no:cacheprovider > gpurun_out/pytest_tc.txt 2>&1; tail -3 gpurun_out/pytest_tc.txt
timeout 900 python -m pytest tests/test_gpu_stream.py -q -rf -s -p no:cacheprovider > gpurun_out/pytest_stream.txt 2>&1; tail -3 gpurun_out/pytest_stream.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -s -p no:cacheprovider -k "fp16ck or mixed" > gpurun_out/pytest_halfck.txt 2>&1; tail -3 gpurun_out/pytest_halfck.txt
[ -n "$TIMING" ] && for sm in direct tc; do MP_SEED_MODE=$sm timeout 300 python scripts/prof_one.py C3 mixed 2 > gpurun_out/c3_mixed_$sm.txt 2>&1; tail -1 gpurun_out/c3_mixed_$sm.txt; done
[ -n "$BENCH" ] && timeout 900 python bench.py --no-per-precision --no-context --no-per-config --no-cpu-baseline > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err; tail -2 gpurun_out/bench_quick.err; cut -c1-300 gpurun_out/bench_quick.json
exit 0
