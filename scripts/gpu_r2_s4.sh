# A/B of library variants on one box: prof_one timing per variant (VARIANTS = lib/exp_<name> dirs,
# "main" = the in-tree library), CASES = "<config>:<precision>" list
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1; tail -1 gpurun_out/build.txt
for rep in 1 2; do
for cfg in ${CASES}; do
  c=${cfg%%:*}; pr=${cfg##*:}
  for v in ${VARIANTS}; do
    if [ "$v" = "main" ]; then lib=""; else lib=$PWD/paper_conf_ipps_juryl022_b200/lib/$v/libmstamp_b200.so; fi
    MP_LIB_PATH=$lib MP_SEED_MODE=${SEED_MODE:-direct} timeout 300 python scripts/prof_one.py $c $pr 1 2>&1 | tail -1 | sed "s/^/$v $cfg: /"
  done
done
done
exit 0
