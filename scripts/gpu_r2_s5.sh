# tests of the half modes / streaming / tensor-core seeds, then C3 timing: direct vs tc seeds
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1; tail -1 gpurun_out/build.txt
timeout 900 python -m pytest tests/test_gpu_stream.py tests/test_gpu_seeds_tc.py -q -rf -s -p no:cacheprovider > gpurun_out/pytest_stream.txt 2>&1; tail -2 gpurun_out/pytest_stream.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -rf -p no:cacheprovider -k "fp16ck or mixed or fp16c" > gpurun_out/pytest_half.txt 2>&1; tail -2 gpurun_out/pytest_half.txt
for sm in direct tc; do for pr in mixed fp16ck; do
  MP_SEED_MODE=$sm timeout 300 python scripts/prof_one.py C3 $pr 1 2>&1 | tail -1 | sed "s/^/$sm C3 $pr: /"
done; done
MP_LIB_PATH=$PWD/paper_conf_ipps_juryl022_b200/lib/exp_base/libmstamp_b200.so timeout 300 python scripts/prof_one.py C3 mixed 1 2>&1 | tail -1 | sed "s/^/base C3 mixed: /"
exit 0
