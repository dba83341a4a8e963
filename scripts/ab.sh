# A/B matrix on one config: env assignments per line of $AB (space-separated VAR=VAL sets, ';'-separated)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
IFS=';' read -ra SETS <<< "${AB:-SAND_PERSIST=1}"
for rep in 1 2; do
for set in "${SETS[@]}"; do
  r=$(env $set timeout 300 python bench.py --config ${CFG:-k400} --steps ${STEPS:-1000} --no-cpu --no-e2e 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('kernel_ms %.4f step_ms %.4f frac %.3f read_us %.1f'%(d['roofline']['kernel_ms_per_step'], d['ms_per_step'], d['roofline']['frac'], d['host']['read_batch_us']), d['host']['kernel_ms_p10_p50_p90'], d['host']['slow_steps'])" 2>&1 | tail -1)
  echo "[$set] $r"
done; done
