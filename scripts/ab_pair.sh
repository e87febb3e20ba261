# A/B of the sweep CTA size (launch bound) for the paired-slot-group sweep
mkdir -p gpurun_out
for t in 1024 768; do
AVFS_NVCC_EXTRA="-DAVFS_SWEEP_THREADS=$t" python -m paper_conf_date_schneiderw20_b200._build > gpurun_out/build$t.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_t$t.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/bench_t$t.log').read().strip().split('\n')[-1]); print('threads $t', round(d['value']/1e9,2), 'Gev/s sweep', round(d['roofline']['kernel_ms'],1), 'ovf', d['stats']['overflow_slot_warps'], 'wpc', d['stats']['warps_per_cta'])"
done
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" 2>&1 | tail -3
t=$(python - <<'P'
import json
a={t: json.loads(open(f'gpurun_out/bench_t{t}.log').read().strip().split('\n')[-1])['roofline']['kernel_ms'] for t in (1024,768)}
print(min(a,key=a.get))
P
)
AVFS_NVCC_EXTRA="-DAVFS_SWEEP_THREADS=$t" python -m paper_conf_date_schneiderw20_b200._build > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sweep -s 1 -c 1 -o gpurun_out/sweep_pair2 -f python scripts/profile_once.py --config 4 > gpurun_out/ncu_pair2.log 2>&1; tail -2 gpurun_out/ncu_pair2.log
