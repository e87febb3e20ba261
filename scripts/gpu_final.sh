# Final round evidence on the committed build: ncu launch list + one full capture of the pass-0
# sweep (config 4), compute-sanitizer, the bench line (with cpu_baseline and e2e), the reference
# arm, the other configs, the whole config 5 on one GPU, and the GPU test suite.
mkdir -p gpurun_out
nproc > gpurun_out/host.txt; grep -m1 "model name" /proc/cpuinfo >> gpurun_out/host.txt
bash scripts/gpu_evidence.sh
timeout 900 python bench.py > gpurun_out/bench_full.log 2>&1; echo bench rc=$?
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.log 2>&1; echo ref rc=$?
bash scripts/gpu_cfgs.sh
timeout 1200 python bench.py --config 5 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg5_full.log 2>&1; echo cfg5full rc=$?
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu_all.log 2>&1; echo pytest rc=$?; tail -1 gpurun_out/pytest_gpu_all.log
