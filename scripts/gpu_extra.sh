# Delay table vs in-sweep evaluation (1-D and the paper's 2-D model) on config 4, and the
# config-5 shard with a capped spill heap (overflow reruns at full size).
mkdir -p gpurun_out
for v in "t0:" "s0:--delay-in-sweep" "t3:--deg-c 3" "s3:--deg-c 3 --delay-in-sweep"; do
  n="${v%%:*}"; a="${v#*:}"
  timeout 900 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e $a > gpurun_out/delay_$n.log 2>&1
  tail -1 gpurun_out/delay_$n.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$n', round(d['ms_per_step'],2), round(d['roofline']['kernel_ms'],2))"
done
timeout 900 python bench.py --config 5 --shard-of 8 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --spill-bytes 30000000000 > gpurun_out/bench_cfg5_overflow.log 2>&1; echo overflow rc=$?
tail -1 gpurun_out/bench_cfg5_overflow.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['overflow'])"
