# Bounds-checked build (-DAVFS_CHECKS: device asserts on the sweep's storage invariants, see
# avfs_kernels.cu) through the GPU test suite and full-size config 4 / config-5 shard / capped-heap
# runs -- the stand-in for compute-sanitizer, which the GPU pool closed.  Rebuilds the normal
# library afterwards.
mkdir -p gpurun_out
AVFS_NVCC_EXTRA=-DAVFS_CHECKS python -c "from paper_conf_date_schneiderw20_b200 import _build; _build.build(force=True)" > gpurun_out/checks_build.log 2>&1; echo build rc=$?
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/checks_pytest.log 2>&1; echo checks pytest rc=$?; tail -1 gpurun_out/checks_pytest.log
timeout 600 python bench.py --config 4 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/checks_cfg4.log 2>&1; echo checks cfg4 rc=$?
timeout 900 python bench.py --config 5 --shard-of 8 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/checks_cfg5.log 2>&1; echo checks cfg5 shard rc=$?
timeout 900 python bench.py --config 5 --shard-of 8 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --spill-bytes 30000000000 > gpurun_out/checks_cfg5_capped.log 2>&1; echo checks cfg5 capped heap rc=$?
timeout 600 python bench.py --config 2 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/checks_cfg2.log 2>&1; echo checks cfg2 rc=$?
python -c "from paper_conf_date_schneiderw20_b200 import _build; _build.build(force=True)" > /dev/null 2>&1; echo rebuild rc=$?
