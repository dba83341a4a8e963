# Full evidence run: GPU tests, smoke, the default bench line (k400, with e2e + cpu_baseline),
# per-config bench lines, reference arm, ncu launch lists and one full capture per config.
# usage: TAG=r02 bash scripts/evidence.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out; T=${TAG:-r02}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv,noheader > gpurun_out/${T}_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; tail -1 gpurun_out/${T}_smoke.log
if [ -z "${SKIP_TESTS:-}" ]; then
  timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/${T}_pytest_gpu.log 2>&1; tail -3 gpurun_out/${T}_pytest_gpu.log
fi
timeout 900 python bench.py > gpurun_out/${T}_bench_default.json 2> gpurun_out/${T}_bench_default.err; tail -c 400 gpurun_out/${T}_bench_default.json; echo
for c in ${CONFIGS:-slowfast slowfast_hd twoview ray tiny}; do
  timeout 900 python bench.py --config $c --no-cpu > gpurun_out/${T}_bench_$c.json 2> gpurun_out/${T}_bench_$c.err
  python -c "import json; d=json.load(open('gpurun_out/${T}_bench_$c.json')); r=d['roofline']; print('$c', round(d['ms_per_step'],4), 'frac', round(r['frac'],3), r['kernel'], {k:round(v['ms_per_launch'],4) for k,v in r['per_kernel'].items()})" || tail -3 gpurun_out/${T}_bench_$c.err
done
timeout 900 python bench.py --impl reference --steps 200 --warmup 3 > gpurun_out/${T}_bench_reference.json 2> gpurun_out/${T}_bench_reference.err; tail -c 300 gpurun_out/${T}_bench_reference.json; echo
for c in ${NCU_CONFIGS:-k400 slowfast slowfast_hd twoview ray}; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_(plain|stream|stencil|direct|copy)" -c 40 --csv --log-file gpurun_out/${T}_launches_$c.csv \
    python bench.py --config $c --steps 30 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/${T}_ncu_launch_$c.err
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_(plain|stream|stencil|direct|copy)" -s 6 -c 2 -o gpurun_out/${T}_prof_$c -f \
    python bench.py --config $c --steps 12 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/${T}_ncu_full_$c.err
  ncu -i gpurun_out/${T}_prof_$c.ncu-rep --page raw --csv > gpurun_out/${T}_ncu_raw_$c.csv 2>/dev/null
  ncu -i gpurun_out/${T}_prof_$c.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/${T}_ncu_sass_$c.csv.gz
  rm -f gpurun_out/${T}_prof_$c.ncu-rep
done
du -sh gpurun_out; ls gpurun_out | head -80
