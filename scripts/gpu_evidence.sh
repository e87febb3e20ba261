# Round evidence: ncu launch list of the bench command, one ncu --set full capture of the pass-0
# sweep on config 4, compute-sanitizer memcheck / racecheck / synccheck on small workloads.
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_cfg4.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_under_ncu.log 2>&1; echo launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/${TAG:-prof_r02} -f python scripts/profile_once.py --config ${CFG:-4} > gpurun_out/ncu_full.log 2>&1; echo ncu rc=$?
# this build's DRAM traffic per sweep launch -> profiles/ncu_sweep_traffic.json, read by the bench
# lines of the same run (roofline.traffic)
python scripts/ncu_summary.py gpurun_out/${TAG:-prof_r02}.ncu-rep --config ${CFG:-4} --tag ${R:-r02} > gpurun_out/ncu_summary.log 2>&1; echo summary rc=$?
cp profiles/ncu_sweep_traffic.json gpurun_out/ 2>/dev/null
# compute-sanitizer (memcheck / racecheck / synccheck via scripts/sanitize_run.py) only when
# AVFS_SANITIZE=1: the GPU pool closed it late in round 2
if [ "${AVFS_SANITIZE:-0}" = 1 ]; then
for tool in memcheck racecheck synccheck; do
timeout 1200 compute-sanitizer --tool $tool --num-cuda-barriers 64 --error-exitcode 9 python scripts/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1; echo $tool rc=$?
tail -3 gpurun_out/sanitize_$tool.log
done
fi
