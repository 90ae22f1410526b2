# bench line (device value + ME/SME kernel times) per build-knob set: FLAGSETS space-separated, commas inside
cd $GRAFT_REPO_ROOT
for flags in ${FLAGSETS:-""}; do
  f="${flags//,/ }"
  FEVES_NVCC_EXTRA="$f" python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
  [ -n "$TESTK" ] && timeout 900 python -m pytest tests -x -q -m gpu -k "$TESTK" 2>&1 | tail -1
  timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e $BARGS 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels_ms']; print('[$f]', round(d['value'],1), 'ms', round(d['ms_per_step'],4), 'me', round(k['me'],4), 'sme', round(k['sme'],4), 'frac', round(d['roofline']['frac'],4))"
done
