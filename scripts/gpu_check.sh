mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
tail -3 gpurun_out/smoke.log
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" -k "not fullsize" > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -30 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench1.log 2>&1; echo bench rc=$?
tail -3 gpurun_out/bench1.log
if [ "$PROF" = "1" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/prof_sweep_cfg4 -f python scripts/profile_once.py --config 4 > gpurun_out/ncu_full.log 2>&1
echo ncu rc=$?
fi
