mkdir -p gpurun_out
timeout 900 python scripts/cap_scan.py 5 4,8 8 > gpurun_out/cap5.log 2>&1; echo cap rc=$?; cat gpurun_out/cap5.log | tail -5
timeout 2400 python -m pytest tests -x -q -m gpu -k fullsize --durations=20 > gpurun_out/pytest_fullsize.log 2>&1; echo fullsize rc=$?
tail -15 gpurun_out/pytest_fullsize.log
