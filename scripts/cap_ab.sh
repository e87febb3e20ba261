# config 4 sweep time vs capacity (spill heap absorbs oversize regions)
for C in ${CAPS:-4 6 8 12}; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --capacity $C > gpurun_out/cap_$C.log 2>&1
  tail -1 gpurun_out/cap_$C.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C=$C value %.4g sweep %.2f ms frac %.4f' % (d['value'], d['roofline']['kernel_ms'], d['roofline']['frac']), d['stats'])"
done
