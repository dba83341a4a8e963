# streaming-kernel variants on the k400 bench: columns per thread (NP) x sub-band rows (S) x super-band (SB)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for NP in 1 2; do for SB in ${SBS:-56 112}; do for S in ${SS:-4 8 16}; do
  r=$(SAND_STREAM_NP=$NP SAND_STREAM_SB=$SB SAND_STREAM_S=$S timeout 300 python bench.py --config ${CFG:-k400} --steps 1000 --no-cpu --no-e2e 2>/dev/null | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('%.4f %.3f'%(d['roofline']['kernel_ms_per_step'], d['roofline']['frac']))")
  echo "NP=$NP SB=$SB S=$S kernel_ms frac: $r"
done; done; done
