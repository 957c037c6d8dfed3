mkdir -p gpurun_out
MP_BENCH_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus 2 --steps 2 --warmup 3 --backend gloo --no-per-precision > gpurun_out/multirank.txt 2>&1
MP_BENCH_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29532 bench.py --gpus 2 --steps 2 --warmup 3 --backend gloo --no-per-precision --precision fp64 >> gpurun_out/multirank.txt 2>&1
MP_BENCH_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 --impl reference >> gpurun_out/multirank.txt 2>&1
tail -20 gpurun_out/multirank.txt
