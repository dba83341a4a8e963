cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity_r2.py -m gpu -q -x > gpurun_out/pytest_r2h.log 2>&1; tail -3 gpurun_out/pytest_r2h.log
for lib in libsand.so libsand_sb.so; do
  for c in k400 slowfast_hd; do
    SAND_LIB=$lib timeout 600 python bench.py --config $c --no-cpu --no-e2e --steps 1000 > gpurun_out/ab_${lib}_$c.json 2> gpurun_out/ab_${lib}_$c.err
    python -c "import json; d=json.load(open('gpurun_out/ab_${lib}_$c.json')); r=d['roofline']; print('$lib $c', round(d['ms_per_step'],4), 'frac', round(r['frac'],3), r['kernel'], {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" || tail -3 gpurun_out/ab_${lib}_$c.err
  done
done
