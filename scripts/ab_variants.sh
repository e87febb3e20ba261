# A/B of compile-time variants: VARIANTS="name1:flags1;name2:flags2" (flags space-separated)
mkdir -p gpurun_out
IFS=';' read -ra VS <<< "$VARIANTS"
for v in "${VS[@]}"; do
  name="${v%%:*}"; flags="${v#*:}"
  AVFS_NVCC_EXTRA="$flags" python -m paper_conf_date_schneiderw20_b200._build > gpurun_out/build_$name.log 2>&1 || { echo "$name build failed"; continue; }
  timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e ${BENCH_ARGS} > gpurun_out/bench_$name.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/bench_$name.log').read().strip().split('\n')[-1]); print('$name', round(d['value']/1e9,2), 'Gev/s sweep', round(d['roofline']['kernel_ms'],1), 'frac', round(d['roofline']['frac'],3), 'ovf', d['stats']['overflow_slot_warps'], 'wpc', d['stats']['warps_per_cta'], 'grid', d['stats']['grid'])" || tail -3 gpurun_out/bench_$name.log
  if [ "$TESTS" = "1" ]; then timeout 900 python -m pytest tests -x -q -m gpu -k "not fullsize" 2>&1 | tail -2; fi
done
