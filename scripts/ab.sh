# A/B of in-tree library variants: LIBS="base a b" CONFIGS="k400" bash scripts/ab.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in ${CONFIGS:-k400}; do for l in ${LIBS-base}; do
  SAND_LIB=libsand_$l.so timeout 300 python bench.py --config $c --no-cpu --no-e2e ${BENCH_ARGS:-} > gpurun_out/ab_${l}_$c.json 2> gpurun_out/ab_${l}_$c.err
  python -c "import json; d=json.load(open('gpurun_out/ab_${l}_$c.json')); r=d['roofline']; print('$l $c', round(d['ms_per_step'],4), 'frac', round(r['frac'],3), {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" || tail -3 gpurun_out/ab_${l}_$c.err
done; done
if [ -n "${TESTLIB:-}" ]; then SAND_LIB=libsand_$TESTLIB.so timeout 900 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS:-} 2>&1 | tail -3; fi
