# usage: bash scripts/gpu_check.sh [tests] [bench] [ncu]   (env: CONFIGS, NCU_CONFIGS, BENCH_ARGS)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv,noheader
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
if [[ " $* " == *" tests "* ]]; then
  timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -15 gpurun_out/pytest_gpu.log
fi
if [[ " $* " == *" bench "* ]]; then
  for c in ${CONFIGS:-k400}; do
    timeout 900 python bench.py --config $c ${BENCH_ARGS:-} > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -2 gpurun_out/bench_$c.err; cat gpurun_out/bench_$c.json
  done
fi
if [[ " $* " == *" ncu "* ]]; then
  for c in ${NCU_CONFIGS:-k400}; do
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_(stream|stencil|resample)" -c 40 --csv --log-file gpurun_out/launches_$c.csv \
      python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/ncu_launch_$c.err
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_ -s 10 -c 2 -o gpurun_out/prof_$c -f \
      python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/ncu_full_$c.err
    tail -2 gpurun_out/ncu_full_$c.err
  done
fi
