for v in "base:0:" "sorted:1:" "rgm:0:-DAVFS_REG_GROUP_MAJOR=1" "sorted_rgm:1:-DAVFS_REG_GROUP_MAJOR=1"; do
  name=$(echo $v | cut -d: -f1); srt=$(echo $v | cut -d: -f2); fl=$(echo $v | cut -d: -f3)
  AVFS_NVCC_EXTRA="$fl" python -c "from paper_conf_date_schneiderw20_b200 import _build; _build.build(force=True)" > /dev/null 2>&1
  for c in 4 3; do
    AVFS_SORTED_BUFFERS=$srt timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/x_${name}_$c.log 2>&1
    tail -1 gpurun_out/x_${name}_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name cfg $c', round(d['ms_per_step'],2), round(d['roofline']['kernel_ms'],2))"
  done
done
