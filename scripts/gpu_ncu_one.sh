# ncu --set full capture of the main kernel of one config: NCU_CASE=X64_32768_256:fp32 NCU_TAG=... bash scripts/gpu_ncu_one.sh
mkdir -p gpurun_out
pc=${NCU_CASE:-X64_32768_256:fp32}; tag=${NCU_TAG:-$(echo $pc | tr ':' '_')}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s ${NCU_SKIP:-1} -c 1 -o gpurun_out/full_$tag python scripts/prof_one.py ${pc%%:*} ${pc##*:} 1 > gpurun_out/ncu_$tag.log 2>&1
tail -3 gpurun_out/ncu_$tag.log
