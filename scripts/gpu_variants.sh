# time experimental library variants (scripts/build_variant.sh) on the same box
mkdir -p gpurun_out; rm -f gpurun_out/variants.txt
for v in ${VARIANTS:-exp_base exp_mb4 exp_u2 exp_mb4u2}; do
  export MP_LIB_PATH=$PWD/paper_conf_ipps_juryl022_b200/lib/$v/libmstamp_b200.so
  echo "== $v" >> gpurun_out/variants.txt
  for c in ${CASES:-"C2 fp32"}; do timeout 300 python scripts/prof_one.py $c 2 >> gpurun_out/variants.txt 2>&1; done
done
cat gpurun_out/variants.txt
