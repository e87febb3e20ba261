# full bench line (cpu_baseline + e2e) on config ${CFG:-4}
mkdir -p gpurun_out
timeout 1200 python bench.py --config ${CFG:-4} ${BENCH_ARGS} > gpurun_out/bench_full.log 2>&1; echo bench rc=$?
tail -n1 gpurun_out/bench_full.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('value %.4g ms %.2f sweep %.2f frac %.4f e2e %.4g traffic %s cpu %.3g' % (d['value'], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['e2e']['value'], d['roofline']['traffic'], d['cpu_baseline']['value'] if d.get('cpu_baseline') else 0))"
