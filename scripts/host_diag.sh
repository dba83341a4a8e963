# host-side diagnostics of the k400 bench: repeat runs, plan threads
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nproc; cat /proc/cpuinfo | grep "model name" | head -1
for PT in 2 2 4 8; do
  SAND_PLAN_THREADS=$PT timeout 300 python bench.py --config ${CFG:-k400} --steps 1000 --no-cpu --no-e2e 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('PT=$PT', 'kernel_ms %.4f step_ms %.4f frac %.3f'%(d['roofline']['kernel_ms_per_step'], d['ms_per_step'], d['roofline']['frac']), d['host'], d['clocks'])"
done
