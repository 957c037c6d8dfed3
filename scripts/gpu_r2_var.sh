# variant timings + fp32 parity on large-d shapes per variant
mkdir -p gpurun_out; rm -f gpurun_out/var_pytest.txt
for v in ${VARIANTS}; do
  echo "== $v" >> gpurun_out/var_pytest.txt
  MP_LIB_PATH=$PWD/paper_conf_ipps_juryl022_b200/lib/$v/libmstamp_b200.so timeout 600 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "${PYTEST_K:-shapes and fp32}" >> gpurun_out/var_pytest.txt 2>&1
  tail -2 gpurun_out/var_pytest.txt
done
bash scripts/gpu_variants.sh
