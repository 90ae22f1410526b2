# ME_OPT_RF_PER_CTA per BASELINE config (full bench path)
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
for c in ${CFGS:-2160p_sa128 1080p_sa64_4rf}; do
  for r in ${RPCS:-0 1 2}; do
    timeout 600 python bench.py --config $c --steps ${STEPS:-30} --warmup 3 --no-cpu-baseline --no-e2e --rf-per-cta $r 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels_ms']; print('$c rpc=$r', round(d['value'],2), 'ms', round(d['ms_per_step'],4), 'me', round(k['me'],4), 'frac', round(d['roofline']['frac'],4))"
  done
done
