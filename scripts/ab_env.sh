# A/B of runtime env knobs: ENVS="name:VAR=val VAR2=val;..." on config(s) CFG (current build)
mkdir -p gpurun_out
IFS=';' read -ra VS <<< "${ENVS}"
for vf in "${VS[@]}"; do
  name="${vf%%:*}"; envs="${vf#*:}"
  for c in ${CFG:-4}; do
    env $envs timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/abe_${name}_cfg$c.log 2>&1
    tail -1 gpurun_out/abe_${name}_cfg$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name cfg $c', 'ms',round(d['ms_per_step'],2),'sweep',round(d['roofline']['kernel_ms'],2),'grid',d['stats']['grid'])" || tail -3 gpurun_out/abe_${name}_cfg$c.log
  done
done
