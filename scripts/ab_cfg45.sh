mkdir -p gpurun_out
IFS=';' read -ra VS <<< "${VARIANTS}"
for vf in "${VS[@]}"; do
  name="${vf%%:*}"; flags="${vf#*:}"
  AVFS_NVCC_EXTRA="$flags" python -c "from paper_conf_date_schneiderw20_b200 import _build; _build.build(force=True)" > gpurun_out/build_$name.log 2>&1 || { echo "build $name failed"; continue; }
  timeout 900 python bench.py --config 5 --shard-of 8 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab5_$name.log 2>&1
  tail -1 gpurun_out/ab5_$name.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name cfg5 shard', 'ms',round(d['ms_per_step'],2),'sweep',round(d['roofline']['kernel_ms'],2))"
  timeout 900 python bench.py --config 4 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab4_$name.log 2>&1
  tail -1 gpurun_out/ab4_$name.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name cfg4', 'ms',round(d['ms_per_step'],2),'sweep',round(d['roofline']['kernel_ms'],2))"
done
