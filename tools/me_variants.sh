# ME kernel variant sweep: each tools/mev_*.so (built with different -D knobs) timed by bench.py,
# then parity-checked with the GPU parity tests through FEVES_LIB.
cd $GRAFT_REPO_ROOT
for f in tools/mev_*.so; do
  for i in 1 2; do
  FEVES_LIB=$PWD/$f python bench.py --steps 40 --warmup 3 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$f', round(d['value'],1), 'fps me', round(d['kernels_ms']['me'],4), 'me_only', round(d['kernels_ms']['me_only_isolated'],4), 'sme', round(d['kernels_ms']['sme'],4), 'int', round(d['kernels_ms']['int_isolated_clean_l2'],4))"
  done
done
if [ -n "$PARITY" ]; then
  for f in tools/mev_*.so; do
    echo "parity $f: $(FEVES_LIB=$PWD/$f timeout 600 python -m pytest tests -x -q -m gpu 2>&1 | tail -1)"
  done
fi
