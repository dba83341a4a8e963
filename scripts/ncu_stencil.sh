cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stencil2 -s 2 -c 1 -o gpurun_out/prof_stencil -f \
  python bench.py --config twoview --steps 6 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/ncu_stencil.err
tail -2 gpurun_out/ncu_stencil.err
