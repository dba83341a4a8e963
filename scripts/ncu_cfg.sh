# one ncu --set full capture of the top kernel of a config: CFG=<config> K=<kernel regex> NAME=<tag>
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:${K:-k_} -s ${SKIP:-4} -c 1 -o gpurun_out/prof_${NAME:-x} -f \
  python bench.py --config ${CFG:-k400} --steps 8 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/ncu_${NAME:-x}.err
tail -1 gpurun_out/ncu_${NAME:-x}.err
