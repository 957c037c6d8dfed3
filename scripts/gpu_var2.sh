mkdir -p gpurun_out; rm -f gpurun_out/variants.txt
for v in ${VARIANTS}; do
  export MP_LIB_PATH=$PWD/paper_conf_ipps_juryl022_b200/lib/$v/libmstamp_b200.so
  echo "== $v" >> gpurun_out/variants.txt
  while read -r c; do [ -n "$c" ] && timeout 300 python scripts/prof_one.py $c 1 >> gpurun_out/variants.txt 2>&1; done <<< "$CASES"
done
cat gpurun_out/variants.txt
