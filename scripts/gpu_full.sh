# Full-size parity + bench (with cpu_baseline) + launch list.  Run under gpurun.
mkdir -p gpurun_out
nproc > gpurun_out/host_cores.txt; lscpu | grep -i "model name" >> gpurun_out/host_cores.txt
timeout 2400 python -m pytest tests -x -q -m gpu -k fullsize --durations=20 > gpurun_out/pytest_fullsize.log 2>&1; echo fullsize rc=$?
tail -25 gpurun_out/pytest_fullsize.log
timeout 900 python bench.py > gpurun_out/bench_full.log 2>&1; echo bench rc=$?
tail -2 gpurun_out/bench_full.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_cfg4.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_under_ncu.log 2>&1; echo launches rc=$?
