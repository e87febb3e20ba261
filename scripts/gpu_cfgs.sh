# short bench lines for configs 2 and 3 (parity-test configs; bench's N=1 workload is config 4)
mkdir -p gpurun_out
for c in ${CFGS:-2 3}; do
timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e ${BENCH_ARGS} > gpurun_out/bench_cfg$c.log 2>&1; echo cfg$c rc=$?
tail -n1 gpurun_out/bench_cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg$c value %.4g ms %.3f sweep %.3f frac %.4f' % (d['value'], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac']), d['stats'])"
done
