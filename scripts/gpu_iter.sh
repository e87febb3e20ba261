# iteration: smoke, GPU suite (stop at first failure), short config-4 bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?; tail -3 gpurun_out/smoke.log
timeout 900 python -m pytest tests -q -m gpu -x ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -25 gpurun_out/pytest_gpu.log
for c in ${BENCH_CFGS:-4}; do
timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg$c.log 2>&1; echo bench cfg$c rc=$?
tail -1 gpurun_out/bench_cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('value',d['value'],'ms',d['ms_per_step'],'sweep',d['roofline']['kernel_ms'],'frac',d['roofline']['frac'],'stats',d['stats'])" || tail -5 gpurun_out/bench_cfg$c.log
done
