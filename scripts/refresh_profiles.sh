# Copy one gpu_final.sh run (gpurun_out/) into tracked summaries under profiles/ (run here, no GPU).
#   TAG=prof_r02c R=r02 bash scripts/refresh_profiles.sh
set -e
R=${R:-r02}; REP=gpurun_out/${TAG:-prof_r02}.ncu-rep
python scripts/ncu_summary.py $REP --config 4 --tag $R > /dev/null
python scripts/ncu_stall_lines.py $REP > profiles/${R}_sweep_cfg4_stall_lines.txt
python scripts/ncu_lines.py $REP > profiles/${R}_sweep_cfg4_source_lines.txt
python scripts/ncu_opcodes.py $REP > profiles/${R}_sweep_cfg4_sass_opcodes.txt
cp gpurun_out/launches_cfg4.csv profiles/${R}_launches_cfg4.csv
python scripts/launch_shares.py gpurun_out/launches_cfg4.csv > profiles/${R}_launch_shares_cfg4.txt
tail -1 gpurun_out/bench_full.log > profiles/${R}_bench_cfg4.json
tail -1 gpurun_out/bench_ref.log > profiles/${R}_bench_reference_cfg4.json
for c in 2 3; do tail -1 gpurun_out/bench_cfg$c.log > profiles/${R}_bench_cfg$c.json; done
tail -1 gpurun_out/bench_cfg5.log > profiles/${R}_bench_cfg5_shard1of8.json
tail -1 gpurun_out/bench_cfg5_full.log > profiles/${R}_bench_cfg5_full_1gpu.json
cp gpurun_out/host.txt profiles/${R}_gpu_box_host.txt
# (compute-sanitizer was closed on the GPU pool late in round 2: keep the last real run's file)
if [ -f gpurun_out/sanitize_memcheck.log ] && ! grep -q "compute-sanitizer is closed" gpurun_out/sanitize_memcheck.log; then
{ for t in memcheck racecheck synccheck; do echo "== compute-sanitizer --tool $t (scripts/sanitize_run.py)"; tail -4 gpurun_out/sanitize_$t.log; done; } > profiles/${R}_compute_sanitizer.txt
fi
tail -3 gpurun_out/pytest_gpu_all.log > profiles/${R}_pytest_gpu_tail.txt
