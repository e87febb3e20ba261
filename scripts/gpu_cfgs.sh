# bench configs 2, 3, 4 and the config-5 shard (no cpu baseline / e2e)
mkdir -p gpurun_out
for c in 2 3 4; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg$c.log 2>&1
  tail -1 gpurun_out/bench_cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg $c', 'ms',round(d['ms_per_step'],2),'sweep',round(d['roofline']['kernel_ms'],2),'frac',round(d['roofline']['frac'],3), 'evals/s %.3e' % d['value'])" || tail -3 gpurun_out/bench_cfg$c.log
done
timeout 900 python bench.py --config 5 --shard-of 8 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg5.log 2>&1
tail -1 gpurun_out/bench_cfg5.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('cfg 5/8', 'ms',round(d['ms_per_step'],2),'sweep',round(d['roofline']['kernel_ms'],2),'frac',round(d['roofline']['frac'],3), 'evals/s %.3e' % d['value'], d['stats'])" || tail -3 gpurun_out/bench_cfg5.log
