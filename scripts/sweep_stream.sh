# parameter sweep of the streaming kernel (env-tunable shape) on the k400 bench
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for SB in ${SBS:-28 32 40 56 75}; do for S in ${SS:-4 8}; do
  r=$(SAND_STREAM_SB=$SB SAND_STREAM_S=$S timeout 300 python bench.py --config ${CFG:-k400} --steps 1000 --no-cpu --no-e2e 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('%.4f %.3f'%(d['roofline']['kernel_ms_per_step'], d['roofline']['frac']))")
  echo "SB=$SB S=$S kernel_ms frac: $r"
done; done
