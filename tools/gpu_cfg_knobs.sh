# BASELINE configs 1-2 (integer ME only) under build knobs: FLAGSETS = space-separated, commas inside a set
cd $GRAFT_REPO_ROOT
for flags in ${FLAGSETS:-""}; do
  f="${flags//,/ }"
  echo "#### flags: $f"
  FEVES_NVCC_EXTRA="$f" python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
  [ -n "$TESTK" ] && timeout 900 python -m pytest tests -x -q -m gpu -k "$TESTK" 2>&1 | tail -2
  for c in ${CFGS:-1080p_sa32 cif}; do
    timeout 300 python bench.py --config $c --steps 200 --warmup 5 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['value'],1), 'ms', round(d['ms_per_step'],5), 'frac', round(d['roofline']['frac'],4))"
  done
done
