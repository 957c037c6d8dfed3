mkdir -p gpurun_out
VARIANTS="exp_pre exp_base" CASES="C2:mixed C2:fp16 X64_32768_256:mixed X256_8192_512:mixed X256_8192_512:fp16" bash scripts/gpu_variants.sh
CS=/usr/local/cuda/bin/compute-sanitizer
for c in "mixed 8 self" "mixed 64 self" "fp16 64 ab"; do
  tag=$(echo $c | tr ' ' '_')
  timeout 900 $CS --tool racecheck --print-limit 20 python scripts/sanitize_case.py $c 160 16 > gpurun_out/sanitize/racecheck5_$tag.txt 2>&1
  echo "racecheck $c rc=$? $(grep -E 'RACECHECK SUMMARY' gpurun_out/sanitize/racecheck5_$tag.txt | tail -1)"
done | tee gpurun_out/sanitize/summary5.txt
for pc in C3:fp32 C3:mixed; do
  tag=$(echo $pc | tr ':' '_')
  timeout 1500 ncu --set full --clock-control none --import-source on -k regex:mp_diag -s 1 -c 1 -o gpurun_out/full_$tag python scripts/prof_one.py ${pc%%:*} ${pc##*:} 1 > gpurun_out/ncu_$tag.log 2>&1
  tail -1 gpurun_out/ncu_$tag.log
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-per-precision --no-per-config --no-context > gpurun_out/bench_under_ncu.txt 2>&1
MP_BENCH_DEVICE=0 timeout 1800 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --backend gloo --dry-run > gpurun_out/dryrun_c4_n2.json 2> gpurun_out/dryrun_c4_n2.err; echo "dryrun rc=$?"; cut -c1-1500 gpurun_out/dryrun_c4_n2.json
