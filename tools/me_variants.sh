cd $GRAFT_REPO_ROOT
for f in tools/mev_*.so; do
  for i in 1 2; do
  FEVES_LIB=$PWD/$f python bench.py --steps 40 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$f', round(d['value'],1), 'fps me', round(d['kernels_ms']['me'],4), 'me_only', round(d['kernels_ms']['me_only_isolated'],4))"
  done
done
