mkdir -p gpurun_out
for w in 8 16 24 32; do
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --warps-per-cta $w > gpurun_out/bench_w$w.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench_w$w.log').read().strip().split('\n')[-1]); print('wpc $w', d['value'], d['roofline']['kernel_ms'], d['stats']['grid'])"
done
