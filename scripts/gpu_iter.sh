# one GPU iteration: parity tests (new first), bench lines, one ncu capture of the top kernel
# usage: TESTS="tests/x.py ..." CONFIGS="k400 ..." NCU="k400" K=k_plain TAG=x bash scripts/gpu_iter.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
if [ -n "${TESTS:-}" ]; then
  timeout ${TEST_TIMEOUT:-1500} python -m pytest $TESTS -m gpu -q -x ${PYTEST_ARGS:-} > gpurun_out/pytest_${TAG:-x}.log 2>&1; tail -15 gpurun_out/pytest_${TAG:-x}.log
fi
for c in ${CONFIGS:-}; do
  timeout 600 python bench.py --config $c --no-cpu --no-e2e ${BENCH_ARGS:-} > gpurun_out/bench_${TAG:-x}_$c.json 2> gpurun_out/bench_${TAG:-x}_$c.err
  python -c "import json,sys; d=json.load(open('gpurun_out/bench_${TAG:-x}_$c.json')); print('$c', round(d['value']), round(d['ms_per_step'],4), 'frac', round(d['roofline']['frac'],3), d['clocks'].get('sm_mhz'))" || tail -3 gpurun_out/bench_${TAG:-x}_$c.err
done
for c in ${NCU:-}; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:${K:-k_} -s ${SKIP:-6} -c 1 -o gpurun_out/prof_${TAG:-x}_$c -f \
    python bench.py --config $c --steps 12 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/ncu_${TAG:-x}_$c.err
  tail -1 gpurun_out/ncu_${TAG:-x}_$c.err
  ncu -i gpurun_out/prof_${TAG:-x}_$c.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/sass_${TAG:-x}_$c.csv.gz
  ncu -i gpurun_out/prof_${TAG:-x}_$c.ncu-rep --page raw --csv 2>/dev/null > gpurun_out/raw_${TAG:-x}_$c.csv
done
