# Round evidence: full GPU test suite, smoke, bench (with cpu_baseline), launch list, ncu full capture.
mkdir -p gpurun_out
nproc > gpurun_out/host_cores.txt; lscpu | grep -i "model name" >> gpurun_out/host_cores.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 2400 python -m pytest tests -q -m gpu --durations=15 > gpurun_out/pytest_gpu_all.log 2>&1; echo pytest rc=$?
tail -20 gpurun_out/pytest_gpu_all.log
timeout 900 python bench.py > gpurun_out/bench_full.log 2>&1; echo bench rc=$?
tail -1 gpurun_out/bench_full.log | cut -c1-600
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.log 2>&1; echo ref rc=$?
tail -1 gpurun_out/bench_ref.log | cut -c1-300
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_cfg4.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_under_ncu.log 2>&1; echo launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/prof_sweep_cfg4 -f python scripts/profile_once.py --config 4 > gpurun_out/ncu_full.log 2>&1; echo ncu rc=$?
# other configs (parity-test configs; config 5 as rank 0's shard of 8)
for c in 2 3; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg$c.log 2>&1; echo cfg$c rc=$?; done
timeout 900 python bench.py --config 5 --shard-of 8 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg5.log 2>&1; echo cfg5 rc=$?
