# time experimental library variants (scripts/build_variant.sh) on the same box:
#   VARIANTS="exp_a exp_b" CASES="C2:fp32 X64_32768_256:mixed" bash scripts/gpu_variants.sh
mkdir -p gpurun_out; rm -f gpurun_out/variants.txt
for v in ${VARIANTS:-exp_base}; do
  export MP_LIB_PATH=$PWD/paper_conf_ipps_juryl022_b200/lib/$v/libmstamp_b200.so
  echo "== $v" >> gpurun_out/variants.txt
  for c in ${CASES:-C2:fp32}; do timeout 300 python scripts/prof_one.py ${c%%:*} ${c##*:} 2 >> gpurun_out/variants.txt 2>&1; done
done
unset MP_LIB_PATH
for c in ${BASE_ONLY_CASES}; do timeout 600 python scripts/prof_one.py ${c%%:*} ${c##*:} 1 >> gpurun_out/variants.txt 2>&1; done
cat gpurun_out/variants.txt
