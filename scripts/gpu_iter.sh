# quick iteration: smoke, GPU parity (not full-size), bench on config 4, optional ncu
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?; tail -3 gpurun_out/smoke.log
timeout 900 python -m pytest tests -x -q -m "gpu" -k "not fullsize" > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -15 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench1.log 2>&1; echo bench rc=$?
tail -1 gpurun_out/bench1.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('value',d['value'],'ms',d['ms_per_step'],'sweep',d['roofline']['kernel_ms'],'frac',d['roofline']['frac'],'ovf',d['stats']['overflow_slot_warps'])"
if [ "$PROF" = "1" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/prof_iter -f python scripts/profile_once.py --config 4 > gpurun_out/ncu_iter.log 2>&1
echo ncu rc=$?; tail -2 gpurun_out/ncu_iter.log
fi
