cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1200 python -m pytest tests -x -q -m gpu 2>&1 | tail -2
for f in tools/mev_*.so; do for c in 2160p_sa128 1080p_sa64_4rf; do
FEVES_LIB=$PWD/$f python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$f $c', round(d['value'],2), 'me', round(d['kernels_ms']['me'],4), 'sme', round(d['kernels_ms']['sme'],4))"
done; done
