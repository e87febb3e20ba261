# one ncu --set full capture of the pass-0 sweep kernel on config ${CFG:-4}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/${TAG:-prof_iter} -f python scripts/profile_once.py --config ${CFG:-4} ${PROF_ARGS} > gpurun_out/ncu_iter.log 2>&1
echo ncu rc=$?; tail -2 gpurun_out/ncu_iter.log
