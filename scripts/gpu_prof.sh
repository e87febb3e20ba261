mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_cfg4.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_under_ncu.log 2>&1
echo launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep -s 1 -c 1 -o gpurun_out/prof_sweep_cfg4 -f python scripts/profile_once.py --config 4 > gpurun_out/ncu_full.log 2>&1
echo ncu rc=$?
tail -5 gpurun_out/ncu_full.log
