mkdir -p gpurun_out; rm -f gpurun_out/variants.txt
for v in exp_base exp_seedsplit; do
  export MP_LIB_PATH=$PWD/paper_conf_ipps_juryl022_b200/lib/$v/libmstamp_b200.so
  echo "== $v" >> gpurun_out/variants.txt
  for c in "C2 fp32" "X64_32768_256 fp32"; do timeout 300 python scripts/prof_one.py $c 1 >> gpurun_out/variants.txt 2>&1; done
done
cat gpurun_out/variants.txt
