mkdir -p gpurun_out
for c in 8 12 16; do
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --capacity $c > gpurun_out/bench_cap$c.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench_cap$c.log').read().strip().split('\n')[-1]); print('cap $c', round(d['value']/1e9,2), 'Gev/s step', round(d['ms_per_step'],1), 'sweep', round(d['roofline']['kernel_ms'],1), 'ovf', d['stats']['overflow_slot_warps'], 'wpc', d['stats']['warps_per_cta'])"
done
