mkdir -p gpurun_out
for d in 0 1; do
AVFS_DYN_GRAB=$d timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_dyn$d.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench_dyn$d.log').read().strip().split('\n')[-1]); print('dyn $d', d['value'], d['roofline']['kernel_ms'], d['stats']['grid'], d['stats']['warps_per_cta'])"
done
