mkdir -p gpurun_out; rm -f gpurun_out/variants.txt
for v in main exp_tg1024 exp_tg512; do
  if [ "$v" = main ]; then export MP_LIB_PATH=; else export MP_LIB_PATH=$PWD/paper_conf_ipps_juryl022_b200/lib/$v/libmstamp_b200.so; fi
  echo "== $v" >> gpurun_out/variants.txt
  for c in "C2 fp32" "C2 mixed" "X64_32768_256 fp32" "X64_32768_256 mixed" "C2 fp64"; do timeout 300 python scripts/prof_one.py $c 1 >> gpurun_out/variants.txt 2>&1; done
done
cat gpurun_out/variants.txt
