# smoke, full GPU suite, short bench on config 4 (no cpu baseline / e2e)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?; tail -2 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu -x --durations=8 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -14 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench1.log 2>&1; echo bench rc=$?
tail -1 gpurun_out/bench1.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('value',d['value'],'ms',d['ms_per_step'],'sweep',d['roofline']['kernel_ms'],'frac',d['roofline']['frac'],'stats',d['stats'])"
