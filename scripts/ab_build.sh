# A/B of compile-time variants: VARIANTS="name:flags;name2:flags2" (flags passed to nvcc), config(s) CFG
mkdir -p gpurun_out
IFS=';' read -ra VS <<< "${VARIANTS}"
for vf in "${VS[@]}"; do
  name="${vf%%:*}"; flags="${vf#*:}"
  AVFS_NVCC_EXTRA="$flags" python -c "from paper_conf_date_schneiderw20_b200 import _build; _build.build(force=True)" > gpurun_out/build_$name.log 2>&1 || { echo "build $name failed"; tail -5 gpurun_out/build_$name.log; continue; }
  for c in ${CFG:-4}; do
    timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab_${name}_cfg$c.log 2>&1
    tail -1 gpurun_out/ab_${name}_cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name cfg $c', 'ms',round(d['ms_per_step'],2),'sweep',round(d['roofline']['kernel_ms'],2),'frac',round(d['roofline']['frac'],3))" || tail -3 gpurun_out/ab_${name}_cfg$c.log
  done
done
