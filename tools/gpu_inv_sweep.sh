cd $GRAFT_REPO_ROOT
for m in 0 16 32 64; do
  FEVES_NVCC_EXTRA="-DFEVES_ME_INV_CF_MAX=$m" python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
  [ $m = 64 ] && timeout 900 python -m pytest tests -x -q -m gpu -k "tiny or rf_per_cta or config2 or pmv or rate_term or sa_inclusive" 2>&1 | tail -1
  for c in cif 1080p_sa32; do
    timeout 300 python bench.py --config $c --steps 200 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('inv<=$m $c', round(d['value'],1), 'frac', round(d['roofline']['frac'],4))"
  done
  timeout 300 python bench.py --steps 60 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('inv<=$m 1080p_s64', round(d['value'],1), 'me', round(d['kernels_ms']['me'],4))"
done
