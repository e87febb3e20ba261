mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
timeout 1200 compute-sanitizer --tool $tool --num-cuda-barriers 64 --error-exitcode 9 python scripts/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1; echo $tool rc=$?
tail -4 gpurun_out/sanitize_$tool.log
done
