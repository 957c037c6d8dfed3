mkdir -p gpurun_out/sanitize
CS=/usr/local/cuda/bin/compute-sanitizer
for c in "fp32 4 self" "fp32 16 self" "fp32 32 ab" "mixed 8 self" "mixed 16 ab" "fp16c 16 self" "fp64 16 self"; do
  tag=$(echo $c | tr ' ' '_')
  timeout 900 $CS --tool racecheck --print-limit 20 python scripts/sanitize_case.py $c 160 16 > gpurun_out/sanitize/racecheck3_$tag.txt 2>&1
  echo "racecheck $c rc=$? $(grep -E 'RACECHECK SUMMARY' gpurun_out/sanitize/racecheck3_$tag.txt | tail -1)"
done | tee gpurun_out/sanitize/summary3.txt
timeout 1800 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/pytest_gpu.txt 2>&1; tail -3 gpurun_out/pytest_gpu.txt
timeout 300 python __graft_entry__.py > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
timeout 1800 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; cut -c1-300 gpurun_out/bench_default.json
# multi-rank path at C4, two ranks sharing this GPU over gloo (functional dry run, not a bench value)
MP_BENCH_DEVICE=0 timeout 2400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --backend gloo --dry-run > gpurun_out/dryrun_c4_n2.json 2> gpurun_out/dryrun_c4_n2.err; echo "dryrun rc=$?"; cut -c1-600 gpurun_out/dryrun_c4_n2.json; tail -3 gpurun_out/dryrun_c4_n2.err
