# session-2: stream / tc tests after fixes; C3 Mixed & FP32 timing base (session start) vs now
# (direct, tc); ncu --set full of the X64 FP32 / Mixed main kernels
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1; tail -1 gpurun_out/build.txt
timeout 900 python -m pytest tests/test_gpu_stream.py tests/test_gpu_seeds_tc.py -q -rf -s -p no:cacheprovider > gpurun_out/pytest_stream.txt 2>&1; tail -3 gpurun_out/pytest_stream.txt
for cfg in ${TIMING_CFGS:-C3:mixed C3:fp32}; do
  c=${cfg%%:*}; pr=${cfg##*:}
  MP_LIB_PATH=$PWD/paper_conf_ipps_juryl022_b200/lib/exp_base/libmstamp_b200.so timeout 300 python scripts/prof_one.py $c $pr 2 2>&1 | tail -1 | sed "s/^/base $cfg: /"
  timeout 300 python scripts/prof_one.py $c $pr 2 2>&1 | tail -1 | sed "s/^/now-direct $cfg: /"
  [ "$pr" = "mixed" ] && MP_SEED_MODE=tc timeout 300 python scripts/prof_one.py $c $pr 2 2>&1 | tail -1 | sed "s/^/now-tc $cfg: /"
done
for pc in ${NCU_CASES}; do
  tag=$(echo $pc | tr ':' '_')
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/full_$tag python scripts/prof_one.py ${pc%%:*} ${pc##*:} 1 > gpurun_out/ncu_$tag.log 2>&1
  tail -1 gpurun_out/ncu_$tag.log
done
exit 0
