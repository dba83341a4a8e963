# Full evidence run: GPU tests, smoke, the default bench line (k400, with e2e + cpu_baseline),
# per-config bench lines, reference arm, ncu launch lists and full captures.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv,noheader > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; cat gpurun_out/bench_default.json
for c in slowfast twoview ray tiny; do
  timeout 900 python bench.py --config $c --no-cpu > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
timeout 900 python bench.py --impl reference --steps 200 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err; cat gpurun_out/bench_reference.json
for c in ${NCU_CONFIGS:-k400 slowfast twoview ray}; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_(stream|stencil|resample|direct|copy)" -c 40 --csv --log-file gpurun_out/launches_$c.csv \
    python bench.py --config $c --steps 30 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/ncu_launch_$c.err
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_(stream|stencil|resample|direct|copy)" -s 6 -c 2 -o gpurun_out/prof_$c -f \
    python bench.py --config $c --steps 12 --warmup 3 --no-e2e --no-cpu > /dev/null 2> gpurun_out/ncu_full_$c.err
  ncu -i gpurun_out/prof_$c.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$c.csv 2>/dev/null
  ncu -i gpurun_out/prof_$c.ncu-rep --page details --csv > gpurun_out/ncu_details_$c.csv 2>/dev/null
  ncu -i gpurun_out/prof_$c.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_sass_$c.csv 2>/dev/null
  gzip -f gpurun_out/ncu_sass_$c.csv
  [ "$c" = "k400" ] || rm -f gpurun_out/prof_$c.ncu-rep
done
du -sh gpurun_out; ls gpurun_out
