mkdir -p gpurun_out
export AVFS_BENCH_SHARE_GPU=1
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --config 3 --steps 3 --warmup 3 > gpurun_out/bench_2rank.log 2>&1; echo 2rank rc=$?
tail -3 gpurun_out/bench_2rank.log | cut -c1-900
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --impl reference --gpus 2 --config 3 --steps 2 --warmup 1 > gpurun_out/bench_2rank_ref.log 2>&1; echo 2rank-ref rc=$?
tail -2 gpurun_out/bench_2rank_ref.log | cut -c1-400
