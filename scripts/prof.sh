# usage: CFGS="k400 slowfast" K=<kernel regex> TAG=<name> bash scripts/prof.sh
# one ncu --set full capture (source-correlated) per config + a SASS source-page export
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in ${CFGS:-k400}; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:${K:-k_} -s ${SKIP:-6} -c 1 -o gpurun_out/prof_${TAG:-x}_$c -f \
    python bench.py --config $c --steps 12 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/ncu_${TAG:-x}_$c.err
  tail -1 gpurun_out/ncu_${TAG:-x}_$c.err
  ncu -i gpurun_out/prof_${TAG:-x}_$c.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/sass_${TAG:-x}_$c.csv.gz
  ncu -i gpurun_out/prof_${TAG:-x}_$c.ncu-rep --page raw --csv 2>/dev/null > gpurun_out/raw_${TAG:-x}_$c.csv
done
