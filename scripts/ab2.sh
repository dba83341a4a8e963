cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for rep in 1 2 3; do
for V in 1024 128 16; do
  r=$(timeout 300 python bench.py --config k400 --videos $V --steps 1000 --no-cpu --no-e2e 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('kernel_ms %.4f step_ms %.4f frac %.3f read_us %.1f'%(d['roofline']['kernel_ms_per_step'], d['ms_per_step'], d['roofline']['frac'], d['host']['read_batch_us']))" 2>&1 | tail -1)
  echo "[V=$V] $r"
done; done
